#!/bin/bash
# u8 Gaussian 5x5 at 4096^2: tile rows x buffering x co-resident CTAs (capped by padding the
# dynamic shared memory, LOP_CONV_SMEM_PAD): does a staggered multi-wave schedule overlap the
# load / compute / store phases that one lock-step wave serialises?  Run under gpurun.
for cfg in 16:1 4:1 32:1 8:2 16:2; do
  for pad in 0 20000 40000 60000 100000; do
    r=$(LOP_CONV_CFG=$cfg LOP_CONV_SMEM_PAD=$pad timeout 120 python tools/time_conv_u8.py 5 2>&1 | tail -1)
    echo "cfg=$cfg pad=$pad $r"
  done
done
