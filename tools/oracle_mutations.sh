#!/bin/bash
# Mutation check of the oracle's pins: apply one plausible mistake at a time to a scratch copy
# of oracle/oracle.c and confirm that tests/test_oracle_pins.py catches it.  CPU only.
# Usage: tools/oracle_mutations.sh      (prints "<label>: N failed, M passed" per mutation)
set -u
REPO=$(cd "$(dirname "$0")/.." && pwd)
run() {
  rm -rf /tmp/orc_mut && mkdir -p /tmp/orc_mut && cp -r "$REPO/oracle" "$REPO/synth" "$REPO/tests" /tmp/orc_mut/
  rm -f /tmp/orc_mut/oracle/liboracle.so
  sed -i "$1" /tmp/orc_mut/oracle/oracle.c
  if cmp -s /tmp/orc_mut/oracle/oracle.c "$REPO/oracle/oracle.c"; then echo "$2: SED DID NOT APPLY"; return; fi
  (cd /tmp/orc_mut && timeout 600 python -m pytest tests/test_oracle_pins.py -q -p no:cacheprovider 2>&1 | tail -1 | sed "s/^/$2: /")
}
run 's/double q\[3\] = {-d\[0\], -d\[1\], 1.0 - d\[2\]};/double q[3] = {d[0], d[1], d[2] - 1.0};/' q_sign
run 's/out\[3 \* i + j\] = (cof\[3 \* j + i\] \/ det)/out[3 * i + j] = (cof[3 * i + j] \/ det)/' transposed_inverse
run 's/double km = 0.5 \* (k1 + k2);/double km = k1;/' midpoint_dropped
run 's/return 1.0 \/ (2.0 \* ORC_PI);/return 1.0;/' dropped_2pi
run 's/if (!(k2 > k1)) continue;/if (!(k2 >= k1)) continue;/' zero_length_segments_kept
run 's/int64_t b = idx\[0\] + c->n\[0\] \* (idx\[1\] + c->n\[1\] \* idx\[2\]);/int64_t b = idx[1] + c->n[1] * (idx[0] + c->n[0] * idx[2]);/' bin_axis_order
run 's/return fF\[lo\] + (fF\[lo + 1\] - fF\[lo\]) \* ((x - fk\[lo\]) \/ (fk\[lo + 1\] - fk\[lo\]));/return fF[lo] + (fF[lo + 1] - fF[lo]) * ((x - fk[lo]) \/ (fk[lo + 1] - fk[0]));/' flux_wrong_index
run 's/for (int64_t j = 1; j < c->n\[a\]; ++j)/for (int64_t j = 1; j < c->n[a] - 1; ++j)/' last_plane_dropped
run 's/double val = (F2 - F1) \* omega_c;/double val = (F2 - F1);/' omega_c_dropped
run 's/lk = c->hi\[a\] \* r;/lk = c->lo[a] * r;/' clip_negative_v
run 's/matmul3(R, UB, A);/matmul3(UB, R, A);/' R_UB_order
run 's/c->w\[a\] = (g->hi\[a\] - g->lo\[a\]) \/ (double)g->n\[a\];/c->w[a] = (g->hi[a] - g->lo[a]) \/ (double)(g->n[a] + 1);/' bin_width
run 's/neu_add(binmd_sum, binmd_comp, b, (double)ev\[col_w\]);/neu_add(binmd_sum, binmd_comp, b, 1.0);/' binmd_weight_dropped
run 's/double x = (N\[3 \* a + 0\] \* q\[0\] + N\[3 \* a + 1\] \* q\[1\]) + N\[3 \* a + 2\] \* q\[2\];/double x = (N[a + 0] * q[0] + N[a + 3] * q[1]) + N[a + 6] * q[2];/' binmd_transposed_N
