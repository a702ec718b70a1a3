#!/bin/bash
O=gpurun_out
L=paper_conf_ipps_ayresc18_b200/_lib
timeout 600 python -m pytest tests/test_gpu_next.py -q -k "dmma" > $O/dmma_tests.log 2>&1; tail -3 $O/dmma_tests.log
for v in "" -psm3 -psm4 -psm5 -psm6; do
  RRL_LIB_PATH=$PWD/$L/librrl$v.so timeout 300 python bench.py --steps 300 --no-cpu-baseline --no-secondary --no-strong > $O/bench_c1$v.json 2>&1
done
for v in "" -psm5; do
  RRL_LIB_PATH=$PWD/$L/librrl$v.so timeout 300 python bench.py --steps 100 --precision 64 --no-cpu-baseline --no-secondary --no-strong > $O/bench_c1_fp64$v.json 2>&1
done
timeout 300 python bench.py --config c3 --precision 64 --steps 10 --no-cpu-baseline --no-secondary --no-strong > $O/bench_c3_fp64.json 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:codon_tc5 -s 0 -c 3 -o $O/prof_c3_tc5 \
  python bench.py --config c3 --steps 1 --warmup 3 --no-cpu-baseline --no-secondary --no-strong --no-graph > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:codon_dmma -s 0 -c 2 -o $O/prof_c3_dmma \
  python bench.py --config c3 --precision 64 --steps 1 --warmup 3 --no-cpu-baseline --no-secondary --no-strong --no-graph > /dev/null 2>&1
for c in c3_tc5 c3_dmma; do
  python tools/ncu_summary.py $O/prof_$c.ncu-rep "$c" > $O/ncu_full_$c.md 2>&1
  ncu -i $O/prof_$c.ncu-rep --page details --csv > $O/ncu_details_$c.csv 2>/dev/null
  ncu -i $O/prof_$c.ncu-rep --page raw --csv > $O/ncu_raw_$c.csv 2>/dev/null
  ncu -i $O/prof_$c.ncu-rep --page source --csv > $O/ncu_source_$c.csv 2>/dev/null
done
rm -f $O/*.ncu-rep
ls -la $O
