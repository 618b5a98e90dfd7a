# developer experiment: time the sequential kernel with one role's work removed
# (SEQ_ABLATE=1 no accounting, 2 no producer math, 3 no recurrence) or with
# another producer count (NPROD)
mkdir -p gpurun_out/s14
for NP in ${NPROD:-6}; do
for A in ${ABL:-0 1 2 3}; do
  MAGUS_NVCC_FLAGS="-DSEQ_ABLATE=$A -DSEQ_NPROD=$NP" python -c "import sys; sys.path.insert(0,'paper_conf_sc_zhengspl25_b200'); import _build; _build.build_libmagus()" > /dev/null 2>&1
  for v in 1 2; do
    timeout 300 python bench.py --variant $v --step 2 --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/s14/b_${A}_${v}.json 2> gpurun_out/s14/b_${A}_${v}.err
    python -c "import json;d=json.load(open('gpurun_out/s14/b_${A}_${v}.json'));print('nprod', $NP, 'ablate', $A, 'variant', $v, d['roofline']['kernel_ms'])" || tail -3 gpurun_out/s14/b_${A}_${v}.err
  done
done
done
