mkdir -p gpurun_out/san
for tool in racecheck synccheck memcheck initcheck; do echo "== $tool"; timeout 1500 compute-sanitizer --tool $tool python tests/sanitize_run.py 2>&1 | grep -E "parity|SUMMARY|Error|error" | head -8; done > gpurun_out/san/summary.txt 2>&1
cat gpurun_out/san/summary.txt
