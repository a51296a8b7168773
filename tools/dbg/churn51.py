import numpy as np, sys
sys.path.insert(0, '.')
import paper_conf_pldi_jablinpjjba11_b200 as cg
import tests.test_gpu_parity as T
from tests.harness import Pair, host_read
from oracle import Oracle
flags = int(sys.argv[1]) if len(sys.argv) > 1 else 0
ctx = cg.Context(0, arena_bytes=1 << 30, flags=flags)
o = Oracle()
P = Pair(ctx, o)
step = [0]
B0 = [None]
def rel(x):
    return hex(x - B0[0]) if B0[0] and x else hex(x)
orig = P.run
def run(name, *a):
    r = orig(name, *a) if False else None
    g = getattr(P.g, name)(*a); P.feed_replay(); oo = getattr(P.o, name)(*a)
    gs = g[0] if isinstance(g, tuple) else g; os_ = oo[0] if isinstance(oo, tuple) else oo
    if step[0] >= 95: print(step[0], name, [rel(x) for x in a[0]], gs, os_)
    return g
P.run = run
sync0 = P.sync_host_to_oracle
def sync(base, n):
    sync0(base, n); step[0] >= 95 and print(step[0], 'CPU rewrites', rel(base), [rel(int(x)) for x in np.frombuffer(host_read(base, n // 8 * 8), dtype=np.uint64)])
P.sync_host_to_oracle = sync
und0 = P.undeclare
def und(b):
    r = und0(b); print(step[0], 'undeclare', rel(b), r); return r
P.undeclare = und
def chk(what=''):
    if B0[0] is None:
        B0[0] = min(u['base'] for u in P.o.dump())
    gd = {u['base']: u for u in P.g.dump()}; od = {u['base']: u for u in P.o.dump()}
    bad = [(rel(b), gd.get(b), od.get(b)) for b in set(gd) | set(od) if gd.get(b) != od.get(b)]
    for b, n in P.units.items():
        hb = np.frombuffer(host_read(b, n // 8 * 8), dtype=np.uint64); ob = P.o.host_read(b, n // 8 * 8).view(np.uint64)
        if (hb != ob).any():
            bad.append(('HOST', rel(b), n, [rel(int(x)) for x in hb], [rel(int(x)) for x in ob]))
    if bad:
        print('DIVERGE at', what)
        for x in bad: print('  ', x)
        for b in sorted(od):
            u = od[b]
            if u['size'] % 8 != 0 or b - B0[0] >= 0x10000 and b - B0[0] < 0x20000:
                print('   outer', rel(b), u['refCount'], [rel(int(x)) for x in np.frombuffer(host_read(b, u['size'] // 8 * 8), dtype=np.uint64)])
        raise SystemExit(1)
    step[0] += 1
P.check = chk
P.check_device_units = lambda *a, **k: None
T._random_array_batches(P, 51, True, churn=True)
print('no divergence')
