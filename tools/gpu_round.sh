#!/bin/bash
# Round artifacts on one B200 (run under gpurun): tests, bench lines, ncu.
# Writes everything to gpurun_out/; summaries are copied to profiles/ by hand.
set -x
O=gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > $O/smi.csv 2>&1
timeout 1500 python -m pytest tests -m gpu -q > $O/gpu_tests.log 2>&1; tail -3 $O/gpu_tests.log
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; tail -2 $O/smoke.log
timeout 900 python bench.py > $O/bench_default.json 2> $O/bench_default.err
timeout 900 python bench.py --impl reference > $O/bench_reference.json 2> $O/bench_reference.err
RRL_DIST_BACKEND=gloo timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 \
  --master-addr 127.0.0.1 --master-port 29511 bench.py --gpus 2 --steps 50 --no-cpu-baseline --no-secondary \
  > $O/bench_2rank_gloo.json 2> $O/bench_2rank_gloo.err
for cfg in c2 c3; do timeout 600 python bench.py --config $cfg --steps 20 --no-cpu-baseline > $O/bench_$cfg.json 2>&1; done
for cfg in c1 c3; do timeout 600 python bench.py --config $cfg --precision 64 --steps 20 --no-cpu-baseline --no-secondary > $O/bench_${cfg}_fp64.json 2>&1; done
timeout 900 python bench.py --config c4 --steps 5 --warmup 3 --no-cpu-baseline > $O/bench_c4.json 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 2000 --csv --log-file $O/launches_default.csv \
  python bench.py --steps 3 --warmup 3 --no-cpu-baseline > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_partials_nuc -s 128 -c 64 \
  -o $O/prof_c1 python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-graph --no-secondary > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_partials_nuc -s 60 -c 20 \
  -o $O/prof_c2_full python bench.py --config c2 --steps 3 --warmup 3 --no-cpu-baseline --no-graph > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:codon_tc -s 54 -c 27 \
  -o $O/prof_c3 python bench.py --config c3 --steps 2 --warmup 3 --no-cpu-baseline --no-graph > /dev/null 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $O/launches_c3.csv \
  python bench.py --config c3 --steps 3 --warmup 3 --no-cpu-baseline > /dev/null 2>&1
# summaries on the box (gpurun copies back at most 64 MiB: the full reports stay here)
for c in c1 c2_full c3; do python tools/ncu_summary.py $O/prof_$c.ncu-rep "$c" > $O/ncu_full_$c.md 2>&1; done
python tools/ncu_traffic.py --out $O/ncu_traffic.json c1_fp32=$O/prof_c1.ncu-rep c2_fp32=$O/prof_c2_full.ncu-rep \
  c3_fp32=$O/prof_c3.ncu-rep > /dev/null 2>&1
python tools/launch_summary.py $O/launches_default.csv > $O/launches_default.md 2>&1
python tools/launch_summary.py $O/launches_c3.csv > $O/launches_c3.md 2>&1
for c in c1 c2_full c3; do
  ncu -i $O/prof_$c.ncu-rep --page details --csv > $O/ncu_details_$c.csv 2>/dev/null
  ncu -i $O/prof_$c.ncu-rep --page raw --csv > $O/ncu_raw_$c.csv 2>/dev/null
done
rm -f $O/*.ncu-rep
timeout 1500 python tools/reroot_sweep.py --out $O/sweep.json > $O/sweep.log 2>&1
du -sh $O; ls -la $O
