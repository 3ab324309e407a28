#!/bin/bash
# usage: tools/sass_fn.sh <lib.so> <mangled-name-substring>  -> SASS of that function
cuobjdump -sass "$1" | awk -v pat="$2" '/Function :/ {on = index($0, pat) > 0} on {print}'
