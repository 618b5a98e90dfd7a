mkdir -p gpurun_out/fin
timeout 300 python bench.py --config 1 --steps 200 --warmup 5 > gpurun_out/fin/bench_cfg1.json 2> gpurun_out/fin/bench_cfg1.err; echo rc1 $?
timeout 900 python bench.py --config 5 --steps 20 --warmup 3 > gpurun_out/fin/bench_cfg5.json 2> gpurun_out/fin/bench_cfg5.err; echo rc5 $?
timeout 1200 python bench.py --config 4 --steps 2 --warmup 3 > gpurun_out/fin/bench_cfg4.json 2> gpurun_out/fin/bench_cfg4.err; echo rc4 $?
python -c "
import json
for f in ('cfg1','cfg5','cfg4'):
  d=json.loads(open('gpurun_out/fin/bench_'+f+'.json').read().strip().splitlines()[-1]); print(f, '%.4g'%d['value'], round(d['ms_per_step'],4), d['config'].get('kernel'), d['roofline']['frac'], d.get('cpu_baseline'), d.get('parity_sample_ok'))
"
