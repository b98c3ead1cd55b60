import gen, paper_conf_ispass_naderantahanse23_b200 as sieve
tr = gen.make_trace("C1")
ctx = sieve.Ctx(device=0)
t = sieve.load_trace(ctx, tr["kid"], tr["x"], num_kernels=tr["K"], cta=tr["cta"], cycles=tr["y"])
st = sieve.stratify(t)
print("ok", len(st))
