#!/bin/bash
# Fused-pass follow-up on one B200 (run under gpurun): full GPU suite, bench
# lines (fused_pass rides along), launch list, ncu --set full of the fused kernel.
set -x
O=gpurun_out
timeout 900 python -m pytest tests -m gpu -q -k fused > $O/fused_tests.log 2>&1; tail -3 $O/fused_tests.log
timeout 600 python bench.py > $O/bench_default_fused.json 2> $O/bench_default_fused.err
timeout 600 python bench.py --precision 64 --steps 50 --no-cpu-baseline --no-secondary > $O/bench_c1_fp64_fused.json 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:k_partials_nuc_fused -s 3 -c 2 \
  -o $O/prof_fused python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-graph --no-secondary > /dev/null 2>&1
python tools/ncu_summary.py $O/prof_fused.ncu-rep c1_fused > $O/ncu_full_c1_fused.md 2>&1
ncu -i $O/prof_fused.ncu-rep --page raw --csv > $O/ncu_raw_c1_fused.csv 2>/dev/null
ncu -i $O/prof_fused.ncu-rep --page source --csv > $O/ncu_source_c1_fused.csv 2>/dev/null
rm -f $O/*.ncu-rep
[ -n "$FULL" ] && timeout 1200 python -m pytest tests -m gpu -q > $O/gpu_tests_full.log 2>&1
ls -la $O
