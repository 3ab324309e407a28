// launch_cache.h -- per-device, thread-safe caches of launch settings.
//
// Kernel attributes (cudaFuncAttributeMaxDynamicSharedMemorySize) and
// occupancy figures belong to a device, and the C ABI runs on whatever device
// is current in the calling thread.  Each cache keeps one slot per device
// ordinal; a slot is an atomic, and computing it twice in racing threads is
// harmless (the CUDA calls are idempotent), so no lock is needed.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include <algorithm>
#include <atomic>

namespace lop {

constexpr int kMaxDevices = 64;

struct PerDevice {
    std::atomic<int64_t> v[kMaxDevices];   // static storage: zero-initialised
    int64_t get(int dev) const
    {
        return dev >= 0 && dev < kMaxDevices ? v[dev].load(std::memory_order_acquire) : 0;
    }
    void set(int dev, int64_t x)
    {
        if (dev >= 0 && dev < kMaxDevices) v[dev].store(x, std::memory_order_release);
    }
};

inline int current_device()
{
    int d = 0;
    cudaGetDevice(&d);
    return d;
}

// Raise `kernel`'s dynamic shared memory limit to `smem` bytes on the current
// device (once per device and size).
template <typename K>
cudaError_t ensure_smem(K kernel, size_t smem, PerDevice &cache)
{
    if (smem <= 48 * 1024) return cudaSuccess;
    const int dev = current_device();
    if ((size_t)cache.get(dev) >= smem) return cudaSuccess;
    const cudaError_t e =
        cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e == cudaSuccess) cache.set(dev, (int64_t)smem);
    return e;
}

// Resident CTAs of `kernel` on the whole current device (SMs x CTAs per SM),
// computed once per device; raises the smem attribute first.  0 on error.
// Both caches must belong to this kernel alone (static at the launcher of one
// template instance: the function-pointer TYPE does not identify a kernel).
template <typename K>
int64_t resident_ctas(K kernel, int threads, size_t smem, PerDevice &smem_cache, PerDevice &cache,
                      cudaError_t &err)
{
    const int dev = current_device();
    int64_t r = cache.get(dev);
    err = cudaSuccess;
    if (r > 0) return r;
    err = ensure_smem(kernel, smem, smem_cache);
    int sms = 0, per_sm = 0;
    if (err == cudaSuccess) err = cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    if (err == cudaSuccess) err = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kernel, threads, smem);
    if (err != cudaSuccess) return 0;
    r = (int64_t)sms * (per_sm > 0 ? per_sm : 1);
    cache.set(dev, r);
    return r;
}

// Resident CTAs of a kernel that allocates `tmem_cols` TMEM columns per CTA
// (tcgen05.alloc; 512 columns per SM): the occupancy API reports 1 CTA per SM
// for such kernels, so the limit is computed from the kernel's registers,
// the shared memory and the TMEM columns (computed once per device).
template <typename K>
int64_t resident_ctas_tmem(K kernel, int threads, size_t smem, int tmem_cols, PerDevice &smem_cache,
                           PerDevice &cache, cudaError_t &err)
{
    const int dev = current_device();
    int64_t r = cache.get(dev);
    err = cudaSuccess;
    if (r > 0) return r;
    err = ensure_smem(kernel, smem, smem_cache);
    if (err != cudaSuccess) return 0;
    cudaFuncAttributes fa;
    int sms = 0, regs_sm = 0, smem_sm = 0, smem_rsv = 0, thr_sm = 0, blk_sm = 0;
    if ((err = cudaFuncGetAttributes(&fa, kernel)) != cudaSuccess ||
        (err = cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev)) != cudaSuccess ||
        (err = cudaDeviceGetAttribute(&regs_sm, cudaDevAttrMaxRegistersPerMultiprocessor, dev)) != cudaSuccess ||
        (err = cudaDeviceGetAttribute(&smem_sm, cudaDevAttrMaxSharedMemoryPerMultiprocessor, dev)) != cudaSuccess ||
        (err = cudaDeviceGetAttribute(&smem_rsv, cudaDevAttrReservedSharedMemoryPerBlock, dev)) != cudaSuccess ||
        (err = cudaDeviceGetAttribute(&thr_sm, cudaDevAttrMaxThreadsPerMultiProcessor, dev)) != cudaSuccess ||
        (err = cudaDeviceGetAttribute(&blk_sm, cudaDevAttrMaxBlocksPerMultiprocessor, dev)) != cudaSuccess)
        return 0;
    const int warps = (threads + 31) / 32;
    const int regs_warp = ((fa.numRegs * 32 + 255) / 256) * 256;       // per-warp allocation unit
    int per_sm = regs_sm / (regs_warp * warps);
    const size_t smem_cta = smem + (size_t)fa.sharedSizeBytes + (size_t)smem_rsv;
    per_sm = std::min(per_sm, (int)((size_t)smem_sm / smem_cta));
    per_sm = std::min(per_sm, 512 / tmem_cols);
    per_sm = std::min(per_sm, thr_sm / threads);
    per_sm = std::min(per_sm, blk_sm);
    r = (int64_t)sms * std::max(per_sm, 1);
    cache.set(dev, r);
    return r;
}

}  // namespace lop
