/*
 * gen_host.c -- host build of the synthetic trace generator (gen/magus_gen.h).
 * Input plumbing only; used by the tests and bench to feed the oracle with the
 * same traces the CUDA generator writes to HBM.
 */
#include <stdint.h>
#include "magus_gen.h"

/* out[t*ld + i] = sample t of trace id0+i;  returns 0, or -1 on bad args */
int magus_gen_traces_host(uint64_t seed, int64_t id0, int64_t n_traces,
                          int64_t n_steps, int64_t ld, int32_t kind, float* out) {
  if (n_traces < 0 || n_steps < 0 || ld < n_traces || !out) return -1;
  if (kind != MG_KIND_MIX && kind != MG_KIND_ADVERSARIAL) return -1;
  for (int64_t i = 0; i < n_traces; ++i) {
    mg_state g;
    mg_init(&g, seed, id0 + i, kind);
    for (int64_t t = 0; t < n_steps; ++t) out[t * ld + i] = (float)mg_step(&g);
  }
  return 0;
}

/* class of trace id (for the recipe statistics in the tests) */
int32_t magus_gen_class_host(uint64_t seed, int64_t global_id, int32_t kind) {
  mg_state g;
  mg_init(&g, seed, global_id, kind);
  return g.cls;
}
