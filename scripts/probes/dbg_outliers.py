import sys, os, subprocess, numpy as np
sys.path[:0] = ['/root/repo', '/root/repo/tests']
import synth, paper_conf_ipps_gowanlockc15_b200 as m
from test_gpu_outliers import with_long_segments, crossing_queries
c = synth.make_config("C1", scale=0.2)
D, L = with_long_segments(c.D, 20, 3, (0.0, 192.0), 30.0, 40.0, -12.0, 12.0)
g = synth.rng(5)
Q = np.ascontiguousarray(np.concatenate([c.Q[:600], crossing_queries(L, g, 100)]))
for d in (0.005,):
    i1 = m.build_index(D); inf = i1.info(); print({k: inf[k] for k in ('n','grid','bins','outlier_rows','outlier_copies','max_extent')})
    r1 = m.search(i1, Q, d)
    os.environ['DTS_OUTLIERS'] = '0'
    out = subprocess.run([sys.executable, '-c', "import sys,numpy as np; sys.path[:0]=['/root/repo','/root/repo/tests']; import paper_conf_ipps_gowanlockc15_b200 as m; D=np.load('/tmp/D.npy'); Q=np.load('/tmp/Q.npy'); i=m.build_index(D); sys.stdout.buffer.write(m.search(i,Q,%r).tobytes())" % d], capture_output=True, env=dict(os.environ))
    np.save('/tmp/D.npy', D); np.save('/tmp/Q.npy', Q)
    out = subprocess.run([sys.executable, '-c', "import sys,numpy as np; sys.path[:0]=['/root/repo','/root/repo/tests']; import paper_conf_ipps_gowanlockc15_b200 as m; D=np.load('/tmp/D.npy'); Q=np.load('/tmp/Q.npy'); i=m.build_index(D); sys.stdout.buffer.write(m.search(i,Q,%r).tobytes())" % d], capture_output=True, env=dict(os.environ))
    r2 = np.frombuffer(out.stdout, dtype=m.RESULT_DTYPE)
    k1 = set(zip(r1['query_id'].tolist(), r1['entry_id'].tolist())); k2 = set(zip(r2['query_id'].tolist(), r2['entry_id'].tolist()))
    print('with copies', len(r1), 'plain', len(r2), 'missing', len(k2 - k1), 'extra', len(k1 - k2))
    miss = sorted(k2 - k1)[:20]; print('missing sample', miss, 'outlier rows >=', c.D.shape[0])
    extra = sorted(k1 - k2)[:10]; print('extra sample', extra)
    del os.environ['DTS_OUTLIERS']
