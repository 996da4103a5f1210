"""Times the parts of caqr_factor_host at C4 (1M x 192 fp32): one chunk's
factorization, the combine of S chunk R's, the whole pinned H2D, for S in a list."""
import torch

from paper_conf_ipps_andersonbdk11_b200 import caqr


def ev_time(fn, reps=5):
    fn()
    torch.cuda.synchronize()
    ts = []
    for _ in range(reps):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        fn()
        b.record()
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    return sorted(ts)[len(ts) // 2]


m, n = 1_000_000, 192
Ah = torch.empty((n, m), pin_memory=True).t()
Ah.copy_(torch.randn(m, n))
A = caqr.colmajor_empty(m, n)
print(f"H2D whole {ev_time(lambda: A.copy_(Ah, non_blocking=True)):.3f} ms")
for S in (8, 12, 16, 24, 32, 48):
    mc = m // S
    Ac = caqr.colmajor_empty(mc, n)
    Ac.copy_(Ah[:mc])
    A0 = Ac.clone()
    R, ws = caqr.caqr_factor(Ac)
    tf = ev_time(lambda: (Ac.copy_(A0), caqr.caqr_factor(Ac, R=R, ws=ws))) - ev_time(lambda: Ac.copy_(A0))
    st = caqr.colmajor_empty(S * n, n)
    st.copy_(torch.triu(torch.randn(S * n, n, device="cuda")))
    s0 = st.clone()
    Rc, cws = caqr.caqr_combine(st, S)
    tc = ev_time(lambda: (st.copy_(s0), caqr.caqr_combine(st, S, R=Rc, ws=cws))) - ev_time(lambda: st.copy_(s0))
    te = ev_time(lambda: caqr.caqr_factor_host(Ah, S, A=A))
    print(f"S={S}: chunk {mc} rows factor {tf:.3f} ms (x S = {tf * S:.2f}), combine {tc:.3f} ms, "
          f"factor_host {te:.3f} ms")
