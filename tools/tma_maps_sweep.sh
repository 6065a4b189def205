#!/bin/bash
# per-GEMM tensor-map cost: R maps, prefetch distance, boxes per stage
for R in 1 64 4096 65536; do
  for pf in 0 8 32; do
    timeout 60 ./tools/tma_maps $R $pf 1 12 4
  done
  timeout 60 ./tools/tma_maps $R 8 2 6 3
done
