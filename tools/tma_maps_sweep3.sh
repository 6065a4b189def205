#!/bin/bash
# bandwidth vs bytes in flight per SM (random 128-row x 128-B boxes; 256-B pairs), L2 promotion 256 B vs none
for promo in 3 0; do
  for st in 2 3 4 6 8 12; do timeout 60 ./tools/tma_maps 4096 8 1 $st 2 $promo 0; done
  for st in 1 2 3 4 6; do timeout 60 ./tools/tma_maps 4096 8 2 $st 1 $promo 0; done
done
