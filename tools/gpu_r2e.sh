#!/bin/bash
O=gpurun_out
L=paper_conf_ipps_ayresc18_b200/_lib
timeout 900 python -m pytest tests/test_gpu_next.py -q -k "codon" > $O/next_codon.log 2>&1; tail -2 $O/next_codon.log
timeout 600 python -m pytest tests/test_gpu_parity.py -q -k "codon" > $O/parity_codon.log 2>&1; tail -2 $O/parity_codon.log
for v in "" -t128 -t512 -t512m3; do
  RRL_LIB_PATH=$PWD/$L/librrl$v.so timeout 300 python bench.py --steps 300 --no-cpu-baseline --no-secondary --no-strong > $O/bench_c1$v.json 2>&1
done
timeout 300 python bench.py --config c3 --steps 30 --no-cpu-baseline --no-secondary --no-strong > $O/bench_c3.json 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $O/launches_c3.csv \
  python bench.py --config c3 --steps 2 --warmup 3 --no-cpu-baseline --no-secondary --no-strong > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:codon_dmma -s 0 -c 2 -o $O/prof_c3_dmma \
  python bench.py --config c3 --precision 64 --steps 1 --warmup 3 --no-cpu-baseline --no-secondary --no-strong --no-graph > /dev/null 2>&1
python tools/ncu_summary.py $O/prof_c3_dmma.ncu-rep c3_dmma > $O/ncu_full_c3_dmma.md 2>&1
ncu -i $O/prof_c3_dmma.ncu-rep --page details --csv > $O/ncu_details_c3_dmma.csv 2>/dev/null
ncu -i $O/prof_c3_dmma.ncu-rep --page source --csv > $O/ncu_source_c3_dmma.csv 2>/dev/null
rm -f $O/*.ncu-rep
ls -la $O
