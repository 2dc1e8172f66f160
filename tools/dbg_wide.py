import sys; sys.path.insert(0, '.')
from tests import gpu_util as G
import oracle
cases = [("c1*c2", [(420, 30), (400, 30)]), ("c1*c2", [(400, 30), (420, 30)]), ("c1*c2", [(600,200),(300,100)]),
         ("c1/c2", [(450, 0), (300, 0)]), ("c1/c2 - c3*c4", [(450, 0), (300, 0), (420, 30), (400, 30)]),
         ("c1/c2", [(300, 0), (300, 0)]), ("c1/c2", [(400, 5), (300, 0)])]
for expr, types in cases:
    for n in (1, 5):
        lead = (1,) if "/" in expr else ()
        host = G.gen_cols(n, types, config=3, nonzero_lead_cols=lead)
        want, P, S = oracle.eval_sum(expr, G.to_oracle(host, types))
        got, gP, gS = G.gpu_sum_string(expr, G.to_gpu(host, types))
        print(expr, types, n, "OK" if got == want else f"BAD got={got[:40]} want={want[:40]}", flush=True)
