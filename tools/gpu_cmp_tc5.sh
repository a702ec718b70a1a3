L=paper_conf_ipps_ayresc18_b200/_lib
for v in "" -b3 -lo2 -b3lo2; do
  RRL_LIB_PATH=$PWD/$L/librrl$v.so timeout 300 python bench.py --config c3 --steps 30 --no-cpu-baseline --no-secondary --no-strong > gpurun_out/bench_c3$v.json 2>&1
  python -c "import json; d=json.load(open('gpurun_out/bench_c3$v.json')); print('$v', d['updatePartials']['ms_per_pass'], d['roofline']['frac'])"
done
