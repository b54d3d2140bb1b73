#!/bin/bash
# A/B of libspecinfer builds in abtest/ on the rows kernel (C3, C4; n = 128 / 256 at B = 8), twice each.
for rep in 1 2; do
for lib in abtest/lib_*.so; do
  echo "== $lib"
  for c in C3 C4; do timeout 120 python tools/attn_probe.py --config $c --layers 2 --iters 10 --lib $lib; done
done
done
