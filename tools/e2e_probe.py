"""Where does the e2e step time go?  load-only, compute-only, sequential and threaded pipelines."""
import os, sys, time, threading
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import gen
import paper_conf_ispass_naderantahanse23_b200 as sieve

cfg = gen.get_config("C4")
g = gen.Generator(cfg)
n = cfg.n
pin = lambda k, dt: torch.empty(k, dtype=dt, pin_memory=True)
h = {"kid": pin(n, torch.int32), "x": pin(n, torch.int64), "cta": pin(n, torch.int32), "y": pin(n, torch.int64)}
hn = {"kid": h["kid"].numpy().view(np.uint32), "x": h["x"].numpy().view(np.uint64),
      "cta": h["cta"].numpy().view(np.uint32), "y": h["y"].numpy().view(np.uint64)}
g.fill(0, n, out=hn)
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
c1, c2 = sieve.Ctx(device=0, stream=s1), sieve.Ctx(device=0, stream=s2)
T = lambda: time.perf_counter()
def load(c): return sieve.load_trace(c, hn["kid"], hn["x"], num_kernels=cfg.K, cta=hn["cta"], cycles=hn["y"])
def comp(tr): st = sieve.stratify(tr); sieve.predict(st, tr)
for c in (c1, c2):
    tr = load(c); comp(tr); del tr
torch.cuda.synchronize()
t = T()
for i in range(4): tr = load(c1); del tr
print("load only  ms/step", (T() - t) / 4 * 1e3, flush=True)
tr = load(c1)
t = T()
for i in range(4): comp(tr)
print("comp only  ms/step", (T() - t) / 4 * 1e3, flush=True)
del tr
t = T()
for i in range(4): tr = load(c1); comp(tr); del tr
print("sequential ms/step", (T() - t) / 4 * 1e3, flush=True)
# load on c2 in a thread while c1 computes (resident trace)
tr = load(c1)
t = T()
th = threading.Thread(target=lambda: [load(c2) for _ in range(4)])
th.start(); [comp(tr) for _ in range(4)]; t_c = T() - t; th.join()
print("overlap: 4 comp", t_c * 1e3, "4 loads done at", (T() - t) * 1e3, flush=True)
del tr
lock = threading.Lock(); log = []
def worker(c, k):
    for _ in range(k):
        with lock:
            a = T(); tr = load(c); b = T()
        comp(tr); e = T(); del tr
        log.append((c is c1, a - t0, b - t0, e - t0))
t0 = T()
ths = [threading.Thread(target=worker, args=(c, 3)) for c in (c1, c2)]
[x.start() for x in ths]; [x.join() for x in ths]
print("threaded ms/step", (T() - t0) / 6 * 1e3)
for r in sorted(log, key=lambda r: r[1]): print("  ctx1" if r[0] else "  ctx2", "load %.1f-%.1f comp-end %.1f" % tuple(1e3 * v for v in r[1:]))
