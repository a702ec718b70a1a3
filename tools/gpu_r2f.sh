#!/bin/bash
O=gpurun_out
timeout 600 python -m pytest tests/test_gpu_next.py -q -k "dmma" > $O/dmma_tests.log 2>&1; tail -2 $O/dmma_tests.log
timeout 300 python bench.py --config c3 --precision 64 --steps 10 --no-cpu-baseline --no-secondary --no-strong > $O/bench_c3_fp64.json 2>&1
timeout 300 python bench.py --steps 300 --no-cpu-baseline --no-secondary --no-strong > $O/bench_c1.json 2>&1
timeout 300 python bench.py --config c3 --steps 30 --no-cpu-baseline --no-secondary --no-strong > $O/bench_c3.json 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:codon_dmma -s 0 -c 2 -o $O/prof_c3_dmma \
  python bench.py --config c3 --precision 64 --steps 1 --warmup 3 --no-cpu-baseline --no-secondary --no-strong --no-graph > /dev/null 2>&1
python tools/ncu_summary.py $O/prof_c3_dmma.ncu-rep c3_dmma > $O/ncu_full_c3_dmma.md 2>&1
ncu -i $O/prof_c3_dmma.ncu-rep --page details --csv > $O/ncu_details_c3_dmma.csv 2>/dev/null
rm -f $O/*.ncu-rep
timeout 2400 python -m pytest tests -m gpu -q > $O/gpu_tests.log 2>&1; tail -3 $O/gpu_tests.log
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; tail -4 $O/smoke.log
for t in memcheck racecheck synccheck; do timeout 900 compute-sanitizer --tool $t python tools/sanitize.py > $O/sanitize_$t.log 2>&1; tail -2 $O/sanitize_$t.log; done
ls -la $O
