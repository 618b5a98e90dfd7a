# The round's profiling pass on one B200 (run under gpurun): every bench line,
# the launch list and the ncu captures the profiles/ summaries come from.
set -x
O=${OUT:-gpurun_out/r2final}
mkdir -p $O
python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.limit --format=csv > $O/gpu.txt 2>&1
python bench.py --steps 20 --warmup 5 > $O/bench_cfg2.json 2> $O/bench_cfg2.err
python bench.py --steps 20 --warmup 5 --inflight 1 --no-cpu-baseline --no-e2e > $O/bench_cfg2_serial.json 2> $O/bench_cfg2_serial.err
python bench.py --impl reference --steps 20 --warmup 5 > $O/bench_ref_cfg2.json 2> $O/bench_ref_cfg2.err
python bench.py --config 1 --steps 20 --warmup 5 > $O/bench_cfg1.json 2> $O/bench_cfg1.err
python bench.py --config 3 --steps 10 --warmup 3 > $O/bench_cfg3.json 2> $O/bench_cfg3.err
python bench.py --config 5 --steps 10 --warmup 3 > $O/bench_cfg5.json 2> $O/bench_cfg5.err
python bench.py --config 4 --steps 2 --warmup 3 > $O/bench_cfg4.json 2> $O/bench_cfg4.err
T1=$(python -c "import json;print(json.loads(open('$O/bench_cfg5.json').read().strip().splitlines()[-1])['ms_per_step'])")
MAGUS_DIST_BACKEND=gloo timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29511 bench.py --gpus 2 --config 5 --steps 10 --warmup 3 --no-e2e --no-cpu-baseline --t1-ms $T1 > $O/bench_cfg5_gloo2.json 2> $O/bench_cfg5_gloo2.err
MAGUS_DIST_BACKEND=gloo timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29512 bench.py --gpus 2 --config 3 --shard configs --steps 5 --warmup 3 --no-e2e --no-cpu-baseline > $O/bench_cfg3_cfgshard_gloo2.json 2> $O/bench_cfg3_cfgshard_gloo2.err
python bench.py --burst 12000 --steps 100 --warmup 5 --no-cpu-baseline --no-e2e > $O/bench_cfg2_f1.json 2> $O/bench_cfg2_f1.err
python bench.py --bound 8 --steps 5 --warmup 3 > $O/bench_cfg2_f2.json 2> $O/bench_cfg2_f2.err
python bench.py --bound 4 --full-grid --steps 3 --warmup 3 > $O/bench_cfg2_f2full.json 2> $O/bench_cfg2_f2full.err
python bench.py --variant 1 --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > $O/bench_cfg2_f3.json 2> $O/bench_cfg2_f3.err
python bench.py --variant 2 --step 2 --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > $O/bench_cfg2_f4.json 2> $O/bench_cfg2_f4.err
python bench.py --variant 2 --step 2 --steps 10 --warmup 3 --no-cpu-baseline --no-e2e --walk1 1 > $O/bench_cfg2_f4_walk1.json 2> $O/bench_cfg2_f4_walk1.err
python tools_cta_timeline.py --config 2 --reps 4 > $O/timeline_cfg2.json 2>&1
ncu --set full --import-source on --clock-control none -k regex:stream_kernel --launch-skip 3 -c 1 -o $O/prof_cfg2 python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e --inflight 1 > $O/ncu_cfg2.log 2>&1
ncu --set full --import-source on --clock-control none -k regex:family_kernel --launch-skip 8 -c 1 -o $O/prof_cfg3 python bench.py --config 3 --steps 2 --warmup 3 --no-cpu-baseline --no-e2e --inflight 1 > $O/ncu_cfg3.log 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_cfg2.csv python bench.py --steps 20 --warmup 5 --no-cpu-baseline --no-e2e > /dev/null 2>&1
ncu --set full --import-source on --clock-control none -k regex:seq_kernel --launch-skip 3 -c 1 -o $O/prof_cfg2_f3 python bench.py --variant 1 --steps 2 --warmup 3 --no-cpu-baseline --no-e2e --inflight 1 > $O/ncu_cfg2_f3.log 2>&1
ncu --set full --import-source on --clock-control none -k regex:walk_ --launch-skip 9 -c 3 -o $O/prof_cfg2_f4 python bench.py --variant 2 --step 2 --steps 2 --warmup 3 --no-cpu-baseline --no-e2e --inflight 1 > $O/ncu_cfg2_f4.log 2>&1
ncu --set full --import-source on --clock-control none -k regex:bound_ -c 1 -o $O/prof_cfg2_f2 python bench.py --bound 8 --steps 1 --warmup 3 > $O/ncu_cfg2_f2.log 2>&1
ncu --set full --import-source on --clock-control none -k regex:bound_grid -c 1 -o $O/prof_cfg2_f2full python bench.py --bound 4 --full-grid --steps 1 --warmup 3 > $O/ncu_cfg2_f2full.log 2>&1
ls -la $O
