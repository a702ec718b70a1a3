#!/bin/bash
O=gpurun_out
timeout 900 python tools/codon_accuracy.py > $O/codon_accuracy.log 2>&1; tail -8 $O/codon_accuracy.log
timeout 600 python -m pytest tests/test_gpu_next.py -q -k "codon_kernels or unequal" > $O/tcc_tests.log 2>&1; tail -5 $O/tcc_tests.log
for k in tc5 tcc; do RRL_CODON_KERNEL=$k timeout 300 python bench.py --config c3 --steps 20 --no-cpu-baseline --no-secondary --no-strong > $O/bench_c3_$k.json 2>&1; done
RRL_TCC_NMAIN=4 timeout 300 python bench.py --config c3 --steps 20 --no-cpu-baseline --no-secondary --no-strong > $O/bench_c3_tcc4.json 2>&1
RRL_TCC_NMAIN=2 timeout 300 python bench.py --config c3 --steps 20 --no-cpu-baseline --no-secondary --no-strong > $O/bench_c3_tcc2.json 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $O/launches_c3_tcc.csv \
  python bench.py --config c3 --steps 2 --warmup 3 --no-cpu-baseline --no-secondary --no-strong > /dev/null 2>&1
python tools/launch_summary.py $O/launches_c3_tcc.csv > $O/launches_c3_tcc.md 2>&1
ls -la $O
