#!/bin/bash
# Round-end evidence (run under gpurun): GPU tests with recorded parity errors, compute-sanitizer
# over the small cases, ncu captures + launch list + default bench + oracle timing
# (scripts/profile_round.sh), and the Fig. 8/9 ablation.  Summarise with
# `python scripts/write_profiles.py r02`.
OUT=gpurun_out
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
VB_PARITY_OUT=$OUT/parity_final.json timeout 1200 python -m pytest tests -m gpu -q -x > $OUT/gputest_final.log 2>&1
tail -2 $OUT/gputest_final.log
if [ -z "$VB_SKIP_SAN" ]; then   # compute-sanitizer was closed on the round-2 pool late in the round
  VB_SAN_TIMEOUT=420 bash scripts/sanitize.sh $OUT/sanitizer_final > /dev/null 2>&1
  cat $OUT/sanitizer_final/summary.txt
fi
VB_LIB=paper_conf_ppopp_li0yjl19_b200/libvbgemm_cov.so timeout 900 python tests/tools/coverage_check.py > $OUT/coverage_final.jsonl 2>&1
tail -3 $OUT/coverage_final.jsonl
bash scripts/profile_round.sh > $OUT/profile_round.log 2>&1
tail -c 300 $OUT/bench_default.json
timeout 2400 python scripts/ablation.py --out $OUT/ablation_r02.json > $OUT/ablation.log 2>&1
tail -3 $OUT/ablation.log
