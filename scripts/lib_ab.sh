#!/bin/bash
# Process-level A/B of library builds (measurement tool): alternates VB_LIB between the given
# .so files for R rounds, each round one scripts/loads_probe.py run over CASES.
#   bash scripts/lib_ab.sh "C5,N31" 4 libvbgemm.so libvbgemm_variant.so
CASES=$1; R=$2; shift 2
L=paper_conf_ppopp_li0yjl19_b200
for r in $(seq 1 $R); do
  for v in "$@"; do
    VB_LIB=$L/$v timeout 900 python scripts/loads_probe.py $CASES 2>&1 | grep '^{'
  done
done
