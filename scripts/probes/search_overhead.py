"""Per-call fixed cost of dts_search_device on small query sets: device time
(CUDA events around the call), the library's phase times and the number of
kernel launches per call."""
import os, sys, statistics
ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path[:0] = [ROOT]
import torch
import synth
import paper_conf_ipps_gowanlockc15_b200 as m
for name in sys.argv[1:] or ["C1", "C3"]:
    c = synth.make_config(name)
    Dd = torch.from_numpy(c.D).cuda(); Qd = torch.from_numpy(c.Q).cuda()
    s = torch.cuda.current_stream()
    idx = m.build_index_device(Dd, stream=s)
    for tk in (False, True):
        ts = []
        for i in range(30):
            e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
            l0 = m.kernel_launches()
            e0.record(s)
            res, st = m.search_device(idx, Qd, c.d, stream=s, time_kernels=tk)
            e1.record(s)
            torch.cuda.synchronize()
            nl = m.kernel_launches() - l0
            ts.append(e0.elapsed_time(e1))
            res.free()
        print(name, "time_kernels", tk, "median ms", round(statistics.median(ts), 4), "launches", nl,
              {k: round(v, 4) for k, v in st.items() if k.startswith("ms_")}, flush=True)
    # host wall time of the call
    import time
    ws = []
    for i in range(30):
        torch.cuda.synchronize(); t0 = time.perf_counter()
        res, st = m.search_device(idx, Qd, c.d, stream=s)
        torch.cuda.synchronize(); ws.append((time.perf_counter() - t0) * 1e3); res.free()
    print(name, "host wall ms", round(statistics.median(ws), 4), flush=True)
