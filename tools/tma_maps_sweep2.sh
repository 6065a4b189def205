#!/bin/bash
# L2 promotion and delayed 128-B strip pairs
for promo in 0 2 3; do
  timeout 60 ./tools/tma_maps 4096 8 1 12 4 $promo 0
  timeout 60 ./tools/tma_maps 4096 8 2 6 3 $promo 0
  for split in 1 4 16 64; do timeout 60 ./tools/tma_maps 4096 8 1 12 4 $promo $split; done
done
