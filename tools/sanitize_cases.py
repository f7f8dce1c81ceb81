"""Small launches of every kernel family, for compute-sanitizer (memcheck / racecheck /
synccheck / initcheck):

    compute-sanitizer --tool memcheck python tools/sanitize_cases.py

Each case runs one hgemm / hgemm_ex / hgemm_allgather_a call on small ragged shapes
and compares with torch (FP32 reference, loose bound: this is a memory-safety run,
parity is tests/).  Prints one line per case and "ALL OK" at the end."""
import sys

import torch

sys.path.insert(0, ".")
from paper_conf_ipps_00020c20_b200 import binding  # noqa: E402


def run(name, m, n, k, tA, tB, out, beta, cfg=None, compute=None):
    g = torch.Generator(device="cuda").manual_seed(1)
    sa = (k, m) if tA == "T" else (m, k)
    sb = (n, k) if tB == "T" else (k, n)
    A = (torch.rand(sa[1], sa[0], generator=g, device="cuda") * 2 - 1).half()    # stored sa, column-major
    B = (torch.rand(sb[1], sb[0], generator=g, device="cuda") * 2 - 1).half()
    cdt = torch.float32 if out == "f32" else torch.float16
    C0 = (torch.rand(n, m, generator=g, device="cuda") * 2 - 1).to(cdt)
    C = C0.clone()
    binding.set_config(**(cfg or {}))
    try:
        if compute:
            binding.hgemm_ex(m, n, k, 1.0, A, max(1, sa[0]), B, max(1, sb[0]), beta, C, m, tA, tB, out,
                             compute=compute)
        else:
            binding.hgemm(m, n, k, 1.0, A, max(1, sa[0]), B, max(1, sb[0]), beta, C, m, tA, tB, out)
        torch.cuda.synchronize()
        st = binding.get_stats()
    finally:
        binding.set_config()
    opA = A.float() if tA == "T" else A.float().t()       # (m, k)
    opB = B.float().t() if tB == "N" else B.float()       # (k, n)
    ref = (opA @ opB).t() + beta * C0.float()
    err = (C.float() - ref).abs().max().item()
    ok = err <= 0.05 * max(k, 1) ** 0.5
    print(f"{'ok ' if ok else 'BAD'} {name:28s} {m}x{n}x{k} {tA}{tB} {out} beta={beta} -> {st['last_kernel']}"
          f"/{st['block_n']} err {err:.3g}", flush=True)
    return ok


def main():
    ok = True
    shapes = [(300, 520, 200)]
    for tA, tB in (("T", "N"), ("N", "N"), ("N", "T"), ("T", "T")):
        for out in ("f16", "f32"):
            for beta in (0.0, 1.0):
                for kern, bn in (("tc2", 512), ("tc2", 256), ("tc1", 256), ("tc1", 128)):
                    for (m, n, k) in shapes:
                        ok &= run(f"{kern}/{bn}", m, n, k, tA, tB, out, beta, {"kernel": kern, "block_n": bn})
                for bn in (64, 128):
                    for spl in (2, 4, 8):
                        ok &= run(f"splitk/{bn}x{spl}", 96, 300, 1024, tA, tB, out, beta,
                                  {"kernel": "splitk", "block_n": bn, "splits": spl})
                ok &= run("simt", 130, 70, 90, tA, tB, out, beta, {"kernel": "simt"})
    for out in ("f16", "f32"):
        for beta in (0.0, 1.0):
            ok &= run("stream (mt1)", 20000, 96, 512, "T", "N", out, beta, {"kernel": "stream"})
            ok &= run("stream (mt2)", 20000, 200, 512, "T", "N", out, beta, {"kernel": "stream"})
            ok &= run("stream swapped", 64, 3000, 512, "T", "N", out, beta, {"kernel": "stream"})
            ok &= run("stream-K tc2/256", 1100, 1100, 1024, "T", "N", out, beta,
                      {"kernel": "tc2", "block_n": 256, "stream_k": 2})
            ok &= run("stream-K tc1/128", 700, 900, 1024, "T", "N", out, beta,
                      {"kernel": "tc1", "block_n": 128, "stream_k": 2})
            ok &= run("half-tail tc2/512", 1100, 1100, 768, "T", "N", out, beta,
                      {"kernel": "tc2", "block_n": 512, "half_tail": 2, "max_ctas": 12})
            ok &= run("quick return k=0", 100, 100, 0, "T", "N", out, beta)
    for tA, tB in (("T", "N"), ("N", "T")):
        for beta in (0.0, 1.0):
            ok &= run("acc16 auto", 300, 520, 200, tA, tB, "f16", beta, compute="f16")
            ok &= run("acc16 tc2/256", 300, 520, 200, tA, tB, "f16", beta, {"kernel": "tc2", "block_n": 256},
                      compute="f16")
    # fused all-gather, two virtual ranks on this device
    m, n, k = 1024, 520, 256
    g = torch.Generator(device="cuda").manual_seed(3)
    full = (torch.rand(m, k, generator=g, device="cuda") * 2 - 1).half()
    rs = [0, 512, m]
    bufs = [torch.zeros_like(full) for _ in range(2)]
    for q in range(2):
        bufs[q][rs[q]:rs[q + 1]] = full[rs[q]:rs[q + 1]]
    B = (torch.rand(n, k, generator=g, device="cuda") * 2 - 1).half()
    C = torch.zeros(n, m, dtype=torch.float16, device="cuda")
    ws = torch.zeros(8, dtype=torch.int32, device="cuda")
    binding.hgemm_allgather_a(m, n, k, 1.0, bufs[1], k, bufs, rs, 1, B, k, 0.0, C, m, "N", "f16",
                              workspace=ws, chunk_rows=512)
    torch.cuda.synchronize()
    err = (C.float() - (full.float() @ B.float().t()).t()).abs().max().item()
    agok = torch.equal(bufs[1], full) and err < 0.05 * k ** 0.5
    print(f"{'ok ' if agok else 'BAD'} allgather virtual 2 ranks err {err:.3g}", flush=True)
    ok &= agok
    print("ALL OK" if ok else "FAILURES", flush=True)
    return 0 if ok else 1


if __name__ == "__main__":
    sys.exit(main())
