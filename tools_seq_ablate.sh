# developer experiment: time the sequential kernel with roles' work removed
# (SEQ_ABLATE bit mask: 1 no accounting, 2 no producer math, 4 no recurrence,
# 8 no producer loads)
O=${OUT:-gpurun_out/seqabl}
mkdir -p $O
for A in ${ABL:-0 1 4 5 7 13 15}; do
  MAGUS_NVCC_FLAGS="-DSEQ_ABLATE=$A" python -c "import sys; sys.path.insert(0,'paper_conf_sc_zhengspl25_b200'); import _build; _build.build_libmagus()" > /dev/null 2>&1
  for v in ${VARIANTS:-1}; do
    timeout 300 python bench.py --variant $v --step 2 --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > $O/b_${A}_${v}.json 2> $O/b_${A}_${v}.err
    python -c "import json;d=json.load(open('$O/b_${A}_${v}.json'));print('ablate', $A, 'variant', $v, d['roofline'].get('kernel_ms'), d['ms_per_step'])" || tail -3 $O/b_${A}_${v}.err
  done
done
