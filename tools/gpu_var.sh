#!/bin/bash
# Compare compile-time variants (exp/<name>/libgpumem.so) on per-stage device times.
# Usage: tools/gpu_var.sh "cfg1 cfg2" var1 var2 ...   (var "main" = the in-tree library)
CFGS=$1; shift
for v in "$@"; do for c in $CFGS; do
  if [ "$v" = main ]; then LIB=""; else LIB=exp/$v/libgpumem.so; fi
  echo -n "[$v] "; GPUMEM_LIB=$LIB timeout 300 python tools/stage_cmp.py $c radix_bits=0 2>&1 | tail -1
done; done
