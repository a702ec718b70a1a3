L=paper_conf_ipps_ayresc18_b200/_lib
for rep in 1 2; do
for v in "" -pdle -u2; do
  RRL_LIB_PATH=$PWD/$L/librrl$v.so timeout 300 python bench.py --steps 300 --no-cpu-baseline --no-secondary --no-strong > gpurun_out/bench_c1$v.json 2>&1
  python -c "import json; d=json.load(open('gpurun_out/bench_c1$v.json')); print('$v', d['updatePartials']['ms_per_pass'], d['reroot']['updatePartials_speedup'])"
done
done
