#!/bin/bash
# Round artifacts on one B200 (run under gpurun): tests, bench lines, ncu, sanitizers, experiments.
# Writes everything to gpurun_out/; summaries are copied to profiles/ (r02_*) by hand.
set -x
O=gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > $O/smi.csv 2>&1
timeout 2400 python -m pytest tests -m gpu -q > $O/gpu_tests.log 2>&1; tail -3 $O/gpu_tests.log
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; tail -4 $O/smoke.log
timeout 900 python bench.py > $O/bench_default.json 2> $O/bench_default.err
timeout 900 python bench.py --impl reference > $O/bench_reference.json 2> $O/bench_reference.err
# the multi-rank path on one GPU: --gpus 2 re-launches itself under torch.distributed.run (gloo: NCCL refuses two ranks on one device)
RRL_DIST_BACKEND=gloo timeout 900 python bench.py --gpus 2 --steps 50 --no-cpu-baseline --no-secondary \
  > $O/bench_2rank_gloo.json 2> $O/bench_2rank_gloo.err
for cfg in c2 c3; do timeout 600 python bench.py --config $cfg --steps 30 --no-cpu-baseline --no-secondary --no-strong > $O/bench_$cfg.json 2>&1; done
for cfg in c1 c3; do timeout 600 python bench.py --config $cfg --precision 64 --steps 30 --no-cpu-baseline --no-secondary --no-strong > $O/bench_${cfg}_fp64.json 2>&1; done
timeout 900 python bench.py --config c4 --steps 5 --warmup 3 --no-cpu-baseline --no-strong > $O/bench_c4.json 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 3000 --csv --log-file $O/launches_default.csv \
  python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-secondary --no-strong > /dev/null 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $O/launches_c3.csv \
  python bench.py --config c3 --steps 3 --warmup 3 --no-cpu-baseline --no-secondary --no-strong > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_partials_nuc -s 64 -c 64 \
  -o $O/prof_c1 python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-graph --no-secondary --no-strong > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_partials_nuc -s 40 -c 20 \
  -o $O/prof_c2_full python bench.py --config c2 --steps 2 --warmup 3 --no-cpu-baseline --no-graph --no-secondary --no-strong > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:partials_codon -s 54 -c 27 \
  -o $O/prof_c3 python bench.py --config c3 --steps 2 --warmup 3 --no-cpu-baseline --no-graph --no-secondary --no-strong > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:partials_codon -s 54 -c 4 \
  -o $O/prof_c3_fp64 python bench.py --config c3 --precision 64 --steps 1 --warmup 3 --no-cpu-baseline --no-graph --no-secondary --no-strong > /dev/null 2>&1
for c in c1 c2_full c3 c3_fp64; do python tools/ncu_summary.py $O/prof_$c.ncu-rep "$c" > $O/ncu_full_$c.md 2>&1; done
python tools/ncu_traffic.py --out $O/ncu_traffic.json c1_fp32=$O/prof_c1.ncu-rep c2_fp32=$O/prof_c2_full.ncu-rep \
  c3_fp32=$O/prof_c3.ncu-rep c3_fp64=$O/prof_c3_fp64.ncu-rep > /dev/null 2>&1
python tools/launch_summary.py $O/launches_default.csv > $O/launches_default.md 2>&1
python tools/launch_summary.py $O/launches_c3.csv > $O/launches_c3.md 2>&1
for c in c1 c2_full c3 c3_fp64; do
  ncu -i $O/prof_$c.ncu-rep --page details --csv > $O/ncu_details_$c.csv 2>/dev/null
done
rm -f $O/*.ncu-rep
for t in memcheck racecheck synccheck; do timeout 900 compute-sanitizer --tool $t python tools/sanitize.py > $O/sanitize_$t.log 2>&1; done
timeout 900 python tools/codon_accuracy.py > $O/codon_accuracy.log 2>&1
timeout 1500 python tools/paper_experiments.py --trees 1000 --budget-s 700 > $O/paper_experiments.log 2>&1
timeout 1200 python tools/search_loop.py --moves 300 > $O/search_loop.log 2>&1
du -sh $O; ls -la $O
