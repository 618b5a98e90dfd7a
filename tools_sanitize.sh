# compute-sanitizer over tests/sanitize_run.py (run under gpurun); writes $OUT/sanitizers.txt
O=${OUT:-gpurun_out/san}
mkdir -p $O
{
  echo "python tests/sanitize_run.py: $(timeout 600 python tests/sanitize_run.py 2>&1 | tail -1)"
  for t in memcheck racecheck synccheck initcheck; do
    echo "compute-sanitizer --tool $t: $(timeout 1500 compute-sanitizer --tool $t python tests/sanitize_run.py 2>&1 | grep -E 'ERROR SUMMARY|RACECHECK SUMMARY|parity' | tr '\n' ' ')"
  done
} > $O/sanitizers.txt 2>&1
cat $O/sanitizers.txt
