#!/bin/bash
O=gpurun_out
timeout 900 python -m pytest tests/test_gpu_next.py -q -k "dmma or codon or update_tree" > $O/next_tests.log 2>&1; tail -3 $O/next_tests.log
timeout 900 python -m pytest tests/test_gpu_parity.py -q -k "codon or c1 or tiny or category" > $O/parity_subset.log 2>&1; tail -3 $O/parity_subset.log
timeout 300 python bench.py --config c3 --precision 64 --steps 10 --no-cpu-baseline --no-secondary --no-strong > $O/bench_c3_fp64.json 2>&1
timeout 300 python bench.py --config c1 --precision 64 --steps 100 --no-cpu-baseline --no-secondary --no-strong > $O/bench_c1_fp64.json 2>&1
timeout 900 python bench.py > $O/bench_default.json 2> $O/bench_default.err; tail -c 300 $O/bench_default.err
timeout 1200 python tools/search_loop.py --moves 300 > $O/search_loop.log 2>&1; tail -3 $O/search_loop.log
timeout 1500 python tools/paper_experiments.py --trees 1000 --budget-s 700 > $O/paper_experiments.log 2>&1; tail -3 $O/paper_experiments.log
ls -la $O
