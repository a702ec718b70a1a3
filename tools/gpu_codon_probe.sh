#!/bin/bash
# Codon K3-TC5 probe (dev, run under gpurun): per-set times, phase traces of the
# widest and a one-op set, and an ncu --set full capture of two launches with the
# raw metrics exported for reading here.
O=gpurun_out
timeout 300 python tools/set_times.py c3 --reps 10 > $O/c3_set_times.json 2>&1
timeout 300 python tools/trace_tc5.py > $O/c3_trace_wide.txt 2>&1
NARROW=$(python -c "
import json; d=json.load(open('$O/c3_set_times.json')); s=[r for r in d['sets'] if r['ops']==1]; print(s[0]['set'] if s else 26)" 2>/dev/null)
timeout 300 python tools/trace_tc5.py 10000 $NARROW > $O/c3_trace_narrow.txt 2>&1
timeout 600 ncu --set full --clock-control none -k regex:k_partials_codon_tc5 -s 27 -c 26 -o $O/prof_tc5 \
  python bench.py --config c3 --steps 1 --warmup 1 --no-cpu-baseline --no-graph --no-secondary --no-strong > /dev/null 2>&1
ncu -i $O/prof_tc5.ncu-rep --page raw --csv > $O/prof_tc5_raw.csv 2>/dev/null
rm -f $O/prof_tc5.ncu-rep
ls -la $O | tail
