#!/bin/bash
# DRAM locality: random 128-row x 128-B boxes vs groups of consecutive boxes along the row
B=./tools/tma_bench
for cols in 512 1024 4096; do
  for cfg in "64 128 1 12 4 0" "64 128 1 12 4 1" "64 128 2 6 3 2" "64 128 4 3 3 2" "64 128 8 2 2 2" "64 32 1 24 4 0" "64 32 4 8 4 2" "64 64 4 6 3 2"; do
    set -- $cfg
    timeout 60 $B $1 $2 $3 $4 8192 4000 $5 $6 $cols
  done
done
