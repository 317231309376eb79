import sys, numpy as np, torch
sys.path.insert(0, '.')
from tests.inputs import desc_for
from oracle import oracle as O
from paper_conf_icpp_masw25_b200 import capgpu as G
d = desc_for(1, P=4, M=2); o = O.Oracle(d); N = o.n; n = 133
rng = np.random.default_rng(43 + N)
g = G.CapGPU.from_config(d, n_servers=n)
A0 = np.abs(np.where(np.arange(N)[:, None] == 0, 0.05, 0.2) * (1 + 0.2 * rng.standard_normal((N, n)))) + 1e-3
T = lambda x: torch.as_tensor(np.ascontiguousarray(x), dtype=torch.float64, device='cuda')
g.set_prior(T(A0))
lo, hi, m = (np.array([k[x] for k in d["knobs"]]) for x in ("f_min", "f_max", "f_min"))
tm = 40 + 160 * rng.random((N, n))
models = [o.model_new() for _ in range(n)]
for step in range(12):
  f = lo[:, None] + (hi - lo)[:, None] * rng.random((N, n))
  a_true = np.where(np.arange(N)[:, None] == 0, 0.05, 0.2)
  p = 300 + np.sum(a_true * f, axis=0) + rng.normal(0, 11, n)
  thr = tm * rng.random((N, n)) * 1.1
  pmin = 300 + a_true[:, 0] @ lo; pmax = 300 + a_true[:, 0] @ hi
  cap = pmin + rng.uniform(-0.1, 1.1, n) * (pmax - pmin)
  out = g.control_step(T(p), T(f), T(thr), T(tm), T(cap))
  torch.cuda.synchronize()
  u = out['u'].cpu().numpy(); st = out['status'].cpu().numpy(); act = out['active'].cpu().numpy(); ah = out['ahat'].cpu().numpy()
  nbad = 0
  for s in range(n):
      o.model_push(models[s], f[:, s], p[s]); aho = o.model_solve(models[s], A0[:, s])
      tho, Ro, rko = o.weights(thr[:, s], tm[:, s])
      beta = p[s] - cap[s] - aho @ f[:, s]
      uo, acto, tie, sto, _ = o.mpc(aho, Ro, beta, lo, hi, m)
      if not np.allclose(u[:, :, s], uo, rtol=1e-9, atol=1e-9):
          nbad += 1
          if nbad < 4:
              print('step', step, 's', s, 'status', st[s], 'act', act[:, s], acto, 'beta', beta, 'beta+a.m', beta + aho @ m, 'theta', tho, 'R', Ro)
              print('  gpu u', u[:, :, s], '\n  ora u', uo, '\n  ahat', ah[:, s], aho)
  print('nbad', nbad, 'of', n)
