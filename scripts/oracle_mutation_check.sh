#!/usr/bin/env bash
# Mutation check of the oracle pins: each plausible mistake (dropped/flipped
# term, wrong index, transposed operand, wrong clip) must make tests/test_oracle.py fail.
set -u
ROOT=$(cd "$(dirname "$0")/.." && pwd)
W=$(mktemp -d)
muts=(
 's/double c = A\[0\] \* A\[0\] + A\[1\] \* A\[1\] + A\[2\] \* A\[2\] - d \* d;/double c = A[0] * A[0] + A[1] * A[1] + A[2] * A[2] + d * d;/'
 's/double beta = A\[0\] \* V\[0\] + A\[1\] \* V\[1\] + A\[2\] \* V\[2\];/double beta = A[0] * V[0] + A[1] * V[1] - A[2] * V[2];/'
 's/if (!(\*ts < \*te))/if (!(*ts <= *te))/'
 's/V\[0\] = B\[0\] - A\[0\]; V\[1\] = B\[1\] - A\[1\]; V\[2\] = B\[2\] - A\[2\];/V[0] = A[0] - B[0]; V[1] = B[1] - A[1]; V[2] = B[2] - A[2];/'
 's/p\[1\] = (1.0 - f) \* s->y_start + f \* s->y_end;/p[1] = (1.0 - f) * s->y_start + f * s->z_end;/'
 's/hi = tau2 < 1.0 ? tau2 : 1.0;/hi = tau2;/'
 's/\*t_e = (1.0 - hi) \* ts + hi \* te;/*t_e = (1.0 - hi) * ts + hi * ts;/'
 's/position_at(q, \*te, pq);/position_at(q, *ts, pq);/'
 's/tau = -beta \/ a;/tau = beta \/ a;/'
 's/if (tau > 1.0) tau = 1.0;//'
 's/double x = A\[0\] + tau \* V\[0\], y = A\[1\] + tau \* V\[1\]/double x = A[0] + tau * V[0], y = A[1] + tau * V[0]/'
 's/\*dmin = sqrt(x \* x + y \* y + z \* z);/*dmin = x * x + y * y + z * z;/'
 's/if (tau < 0.0) tau = 0.0;//'
)
rc=0
for m in "${muts[@]}"; do
  rm -rf "$W/r" && mkdir "$W/r" && cp -r "$ROOT"/{synth,oracle,tests} "$W/r/" && rm -f "$W/r/oracle/liboracle.so"
  sed -i "$m" "$W/r/oracle/oracle.c"
  if cmp -s "$W/r/oracle/oracle.c" "$ROOT/oracle/oracle.c"; then echo "NOT APPLIED: $m"; rc=1; continue; fi
  if (cd "$W/r" && timeout 300 python -m pytest tests/test_oracle.py -q -p no:cacheprovider >/dev/null 2>&1); then
    echo "SURVIVED: $m"; rc=1
  else
    echo "killed:   $m"
  fi
done
rm -rf "$W"
exit $rc
