"""Tiny search with the TMA-staged pass 1 (DTS_WTILE_TMA=32) against the
default pass 1 on C0: same result bytes expected."""
import os, sys
ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path[:0] = [ROOT, os.path.join(ROOT, "tests")]
import synth
import paper_conf_ipps_gowanlockc15_b200 as m
c = synth.make_config(sys.argv[1] if len(sys.argv) > 1 else "C0")
i = m.build_index(c.D)
r = m.search(i, c.Q, c.d)
print("results", r.shape[0], flush=True)
sys.stdout.flush()
open(os.path.join(ROOT, "gpurun_out", "tma_%s.bin" % os.environ.get("DTS_WTILE_TMA", "0")), "wb").write(r.tobytes())
