L=paper_conf_ipps_ayresc18_b200/_lib
timeout 600 python -m pytest tests/test_gpu_next.py -q -k "codon_tc_per_node or local_op or unequal" > gpurun_out/tc5_tests.log 2>&1; tail -2 gpurun_out/tc5_tests.log
for rep in 1 2; do
for v in "" -d_lo1 -stage -d_a3; do
  RRL_LIB_PATH=$PWD/$L/librrl$v.so timeout 300 python bench.py --config c3 --steps 30 --no-cpu-baseline --no-secondary --no-strong > gpurun_out/bench_c3$v.json 2>&1
  python -c "import json; d=json.load(open('gpurun_out/bench_c3$v.json')); print('$v', d['updatePartials']['ms_per_pass'], d['roofline']['frac'])"
done
done
rm -rf build/rrl-trace; timeout 300 python tools/trace_tc5.py 10000 1 > gpurun_out/trace_set1_direct.txt 2>&1
grep -E "phase period|internal:" gpurun_out/trace_set1_direct.txt
