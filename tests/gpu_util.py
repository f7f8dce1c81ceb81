"""Helpers for the GPU parity tests: run the CUDA path through the C ABI on
seeded inputs and compare with the oracle under the north_star (4) rules."""
from __future__ import annotations

import numpy as np

from paper_conf_ipps_00020c20_b200 import inputs


def ulp16(x):
    """One FP16 ulp at |x|: 2^(max(floor(log2|x|), -14) - 10); 2^-24 at 0."""
    a = np.abs(np.asarray(x, dtype=np.float64))
    e = np.floor(np.log2(np.where(a > 0, a, 1.0)))
    e = np.where(a > 0, np.maximum(e, -14), -14)
    return np.ldexp(1.0, (e - 10).astype(np.int64))


def tolerance(r, absab, alpha, beta, c, out, got=None):
    """Elementwise bound of BASELINE.json north_star (4), generalised to alpha/beta:
    1e-3*(|alpha|*(|A||B|)_ij + |beta|*|c_ij|), plus one FP16 ulp for FP16 output
    (taken at the larger of |r| and |got|, which covers a binade edge)."""
    c = np.zeros_like(r) if c is None or beta == 0 else np.asarray(c, dtype=np.float64)
    bound = 1e-3 * (abs(alpha) * absab + abs(beta) * np.abs(c))
    if out == "f16":
        mag = np.abs(r) if got is None else np.maximum(np.abs(r), np.abs(got))
        bound = bound + ulp16(mag)
    return bound


class GpuCase:
    """One hgemm call on device copies of column-major host buffers."""

    def __init__(self, opA, opB, tA, tB, alpha=1.0, beta=0.0, C=None, out="f16", pad=(0, 0, 0),
                 c_fill=np.nan, align=True):
        import torch
        self.torch = torch
        self.m, self.k = opA.shape
        self.n = opB.shape[1]
        self.tA, self.tB, self.alpha, self.beta, self.out = tA, tB, alpha, beta, out
        sa = inputs.stored_shape(self.m, self.k, tA)
        sb = inputs.stored_shape(self.k, self.n, tB)
        # align: round leading dimensions up to 16 bytes (the TMA fast-path precondition)
        up = (lambda x, q: (x + q - 1) // q * q) if align else (lambda x, q: x)
        qc = 4 if out == "f32" else 8
        self.A, self.lda = inputs.store_op(np.asarray(opA, np.float16), tA, ld=up(max(sa[0], 1), 8) + pad[0])
        self.B, self.ldb = inputs.store_op(np.asarray(opB, np.float16), tB, ld=up(max(sb[0], 1), 8) + pad[1])
        self.ldc = up(max(self.m, 1), qc) + pad[2]
        cdt = np.float32 if out == "f32" else np.float16
        if C is None:
            C = np.full((self.m, self.n), c_fill, dtype=cdt)
        self.C_in = inputs.to_colmajor(np.asarray(C, dtype=cdt), self.ldc, fill=cdt(np.nan))
        self.Cmat = np.asarray(C, dtype=np.float64)

    def run_gpu(self, repeat=1, compute=None):
        """Run hgemm() (or hgemm_ex() with `compute` "f32" / "f16") on device copies."""
        from paper_conf_ipps_00020c20_b200 import binding
        torch = self.torch
        dA = torch.from_numpy(self.A.view(np.int16).copy()).cuda()
        dB = torch.from_numpy(self.B.view(np.int16).copy()).cuda()
        cv = self.C_in.view(np.int16) if self.out == "f16" else self.C_in
        outs = []
        for _ in range(repeat):
            dC = torch.from_numpy(cv.copy()).cuda()
            if compute is None:
                binding.hgemm(self.m, self.n, self.k, self.alpha, dA, self.lda, dB, self.ldb, self.beta, dC,
                              self.ldc, self.tA, self.tB, self.out)
            else:
                binding.hgemm_ex(self.m, self.n, self.k, self.alpha, dA, self.lda, dB, self.ldb, self.beta, dC,
                                 self.ldc, self.tA, self.tB, self.out, compute=compute)
            torch.cuda.synchronize()
            h = dC.cpu().numpy()
            if self.out == "f16":
                h = h.view(np.float16)
            outs.append(h)
        self.stats = binding.get_stats()
        return outs[0] if repeat == 1 else outs

    def oracle(self, oracle_mod, nthreads=8):
        c_out, r, ab = oracle_mod.hgemm_ref(self.m, self.n, self.k, self.alpha, self.A, self.lda, self.B,
                                            self.ldb, self.beta, self.C_in, self.ldc, self.tA, self.tB,
                                            self.out, nthreads=nthreads)
        if self.out == "f16":
            c_out = c_out.view(np.float16)
        return c_out, r, ab

    def view(self, flat):
        return inputs.from_colmajor(flat, self.m, self.n, self.ldc)

    def padding(self, flat):
        return np.asarray(flat).reshape(self.ldc, self.n, order="F")[self.m:, :]


def assert_within_tolerance(case, got_flat, r, ab):
    got = case.view(got_flat).astype(np.float64)
    bound = tolerance(r, ab, case.alpha, case.beta, case.Cmat, case.out, got)
    err = np.abs(got - r)
    bad = ~(err <= bound)
    if bad.any():
        idx = np.argwhere(bad)[:5]
        raise AssertionError(f"{bad.sum()} entries out of tolerance, e.g. {idx.tolist()}: got "
                             f"{got[tuple(idx[0])]} want {r[tuple(idx[0])]} bound {bound[tuple(idx[0])]}")
    rel = np.max(err / np.maximum(ab, 1e-30)) if ab.size else 0.0
    return float(rel)
