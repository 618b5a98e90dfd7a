mkdir -p gpurun_out/final
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/final/smoke.log 2>&1; tail -1 gpurun_out/final/smoke.log
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/final/pytest.log 2>&1; tail -1 gpurun_out/final/pytest.log
timeout 600 python bench.py > gpurun_out/final/bench.json 2> gpurun_out/final/bench.err; echo rc $?
timeout 600 python bench.py --impl reference --steps 20 --warmup 3 > gpurun_out/final/ref.json 2> gpurun_out/final/ref.err; echo rc $?
