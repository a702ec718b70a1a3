#!/bin/bash
O=gpurun_out
L=paper_conf_ipps_ayresc18_b200/_lib
timeout 900 python -m pytest tests/test_gpu_next.py -q > $O/next_tests.log 2>&1; tail -3 $O/next_tests.log
timeout 900 python -m pytest tests/test_gpu_parity.py -q -k "codon or partition" > $O/codon_tests.log 2>&1; tail -3 $O/codon_tests.log
timeout 600 python tools/codon_accuracy.py > $O/codon_accuracy.log 2>&1; tail -3 $O/codon_accuracy.log
timeout 300 python bench.py --config c3 --steps 20 --no-cpu-baseline --no-secondary --no-strong > $O/bench_c3.json 2>&1
for v in "" -minb3 -minb2; do
  RRL_LIB_PATH=$PWD/$L/librrl$v.so timeout 300 python bench.py --steps 200 --no-cpu-baseline --no-secondary --no-strong > $O/bench_c1$v.json 2>&1
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $O/launches_c3.csv \
  python bench.py --config c3 --steps 2 --warmup 3 --no-cpu-baseline --no-secondary --no-strong > /dev/null 2>&1
timeout 900 python bench.py > $O/bench_default.json 2> $O/bench_default.err; tail -c 400 $O/bench_default.err
ls -la $O
