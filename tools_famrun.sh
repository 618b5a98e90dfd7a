O=gpurun_out/$1; mkdir -p $O
timeout 300 python -m pytest tests/test_gpu_family.py -q -x --timeout 100 --timeout_method thread > $O/fam.log 2>&1; tail -2 $O/fam.log
timeout 150 python bench.py --config 3 --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > $O/b3.json 2> $O/b3.err; head -c 300 $O/b3.json; echo
timeout 400 ncu --set full --import-source on --clock-control none -k regex:family_kernel --launch-skip 8 -c 1 -o $O/prof_fam python bench.py --config 3 --steps 2 --warmup 3 --no-cpu-baseline --no-e2e --inflight 1 > $O/ncu.log 2>&1; tail -1 $O/ncu.log
