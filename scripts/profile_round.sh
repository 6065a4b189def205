#!/bin/bash
# Round-end evidence on one B200 (run under gpurun): ncu --set full captures of the dominant
# kernel of C5 (headline), C4 (2-SM pair kernel, and its second, 1-SM launch), C2 (FFMA kernel),
# C3 (GoogleNet GEMMs, nb=1), C3i (implicit-GEMM conv, nb=32) and C1 (FFMA, 8 GEMMs),
# the launch list of the default bench command, and the default bench line.  Summarise here
# afterwards with `python scripts/write_profiles.py <tag>`.
set -x
OUT=gpurun_out
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
NCU="ncu --set full --import-source on --clock-control none -c 1"
timeout 900 $NCU -k regex:vb_tc_kernel -o $OUT/prof_C5 -f python scripts/prof_kernel.py --config C5 --policy threshold > $OUT/prof_C5.log 2>&1
timeout 900 $NCU --kernel-name-base mangled -k regex:ILi1ELb1E -o $OUT/prof_C4 -f python scripts/prof_kernel.py --config C4 --policy binary > $OUT/prof_C4.log 2>&1
timeout 900 $NCU --kernel-name-base mangled -k regex:ILi1ELb0E -o $OUT/prof_C4single -f python scripts/prof_kernel.py --config C4 --policy binary > $OUT/prof_C4single.log 2>&1
timeout 600 $NCU -k regex:vb_f32_kernel -o $OUT/prof_C2 -f python scripts/prof_kernel.py --config C2 --policy binary > $OUT/prof_C2.log 2>&1
timeout 600 $NCU -k regex:vb_f32_kernel -o $OUT/prof_C1 -f python scripts/prof_kernel.py --config C1 --policy threshold > $OUT/prof_C1.log 2>&1
timeout 600 $NCU -k regex:vb_tc_kernel -o $OUT/prof_C3i -f python scripts/prof_kernel.py --config C3i --nb 32 > $OUT/prof_C3i.log 2>&1
timeout 600 $NCU -k regex:vb_tc_kernel -o $OUT/prof_C3 -f python scripts/prof_kernel.py --config C3 > $OUT/prof_C3.log 2>&1
timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none --csv python bench.py --steps 3 --warmup 3 --e2e-steps 1 --cpu-seconds 2 > $OUT/launches_c5.csv 2> $OUT/launches_c5.err
timeout 1200 python bench.py > $OUT/bench_default.json 2> $OUT/bench_default.err
timeout 600 python tests/tools/oracle_timing.py > $OUT/oracle_timing.jsonl 2>&1
tail -c 400 $OUT/bench_default.json
