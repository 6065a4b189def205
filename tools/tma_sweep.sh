#!/bin/bash
B=./tools/tma_bench
for foot in 64 8192; do
  for cfg in "64 64 1 16 1 0" "64 64 1 16 1 1" "64 64 1 16 2 0" "64 64 1 16 4 0" "64 64 2 8 1 0" "64 64 8 3 1 0" "64 64 1 16 4 1" "32 64 1 24 4 0" "64 128 1 12 4 0" "64 128 1 12 1 1"; do
    set -- $cfg
    timeout 60 $B $1 $2 $3 $4 $foot 4000 $5 $6
  done
done
