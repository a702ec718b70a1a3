#!/bin/bash
# Quick round-2 GPU check (run under gpurun): new tests, codon parity, smoke, bench.
O=gpurun_out
timeout 1200 python -m pytest tests/test_gpu_next.py -q > $O/next_tests.log 2>&1; tail -3 $O/next_tests.log
timeout 900 python -m pytest tests/test_gpu_parity.py -q -k "codon or partition or tiny" > $O/codon_tests.log 2>&1; tail -3 $O/codon_tests.log
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; tail -3 $O/smoke.log
timeout 900 python bench.py > $O/bench_default.json 2> $O/bench_default.err; tail -c 300 $O/bench_default.err
timeout 600 python bench.py --config c3 --steps 20 --no-cpu-baseline --no-secondary --no-strong > $O/bench_c3.json 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $O/launches_c3.csv \
  python bench.py --config c3 --steps 2 --warmup 3 --no-cpu-baseline --no-secondary --no-strong > /dev/null 2>&1
python tools/launch_summary.py $O/launches_c3.csv > $O/launches_c3.md 2>&1
ls -la $O
