mkdir -p gpurun_out/w5
timeout 900 python -m pytest tests/test_gpu_walk.py -m gpu -x -q > gpurun_out/w5/pytest.log 2>&1; echo "rc $?" >> gpurun_out/w5/pytest.log
for v in "2 --step 2" "2 --step 1"; do timeout 300 python bench.py --variant $v --steps 20 --warmup 3 --no-cpu-baseline --no-e2e >> gpurun_out/w5/bench.json 2>> gpurun_out/w5/bench.err; done
ncu --metrics gpu__time_duration.sum,smsp__inst_executed.sum,smsp__issue_active.avg.pct_of_peak_sustained_active,dram__bytes_read.sum --clock-control none -k regex:walk_ --launch-skip 3 -c 3 --csv python bench.py --variant 2 --step 2 --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/w5/ncu.csv 2>&1
tail -3 gpurun_out/w5/pytest.log
