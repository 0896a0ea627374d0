"""Seeded synthetic image stacks shaped like the paper's workloads.

This module is the ONLY code shared by the CUDA path's tests/bench and the
oracle's tests: it draws inputs and holds none of BFAST-Monitor's
arithmetic (no design matrix, no fit, no MOSUM).  It uses plain torch ops on
whatever device the caller names (PyTorch is plumbing here), so a stack of
26.8 GB can be generated directly in HBM.

Recipe (parameters mimic the Landsat NDMI stacks
of L47/L377 and the Table I structure of L303-L319):
  dates   d_t = year0 + t/f, t = 1..N (f = 23: 16-day Landsat, L53).
  signal  y = a + b (d_t - d_1) + sum_{j=1..3} (u_j sin 2 pi j d_t + w_j cos 2 pi j d_t)
          + eps,  a ~ U[0.3,0.8], b ~ U[-0.01,0.01], u_j, w_j ~ U[-0.1,0.1],
          eps ~ N(0, s^2), s ~ U[0.01,0.05] per pixel.
  breaks  a fraction of pixels gets a step -delta, delta ~ U[0.1,0.5], from
          t0 ~ U{n, ..., N-1} (0-based) on.
  missing "iid": Bernoulli(miss) per (t, p)  (Table I's f_NaN, L309);
          "cloud": per date a cover c_t ~ U[max(0,2m-1), min(1,2m)] and the
          pixels below the c_t-quantile of a smooth value-noise field
          (64-pixel lattice, bilinear) are NaN (cloud masks, L95).
The stack is time-major Y[t][p] with leading dimension ldY >= P (the
paper's Y^T, L185); columns P..ldY-1 are NaN padding.
"""
from __future__ import annotations

import math
from dataclasses import dataclass, asdict

import numpy as np
import torch


@dataclass
class StackSpec:
    P: int
    N: int
    n_hist: int
    k: int = 3
    hf: float = 0.25
    lam: float = 1.65
    miss: float = 0.5
    mask: str = "iid"          # "iid" | "cloud" | "none"
    break_frac: float = 0.1
    f: float = 23.0
    year0: float = 2000.0
    seed: int = 1
    noise_lo: float = 0.01
    noise_hi: float = 0.05
    dense_hist: bool = False   # no missing value before n_hist (the NaN-free case of L93)
    empty_frac: float = 0.0    # share of date slices with no value at all (L379; drawn per date)

    def asdict(self):
        return asdict(self)


# The configs of BASELINE.json (configs[0..4]); n_hist = N/2 where BASELINE is
# silent (as in D1-D5, L319), k = 3, hf = 0.25, lambda = 1.65.
CONFIGS = {
    "tiny": StackSpec(P=4096, N=228, n_hist=114, miss=0.5, mask="iid", break_frac=0.3, seed=1),
    "landsat": StackSpec(P=4096 * 4096, N=400, n_hist=200, miss=0.6, mask="cloud",
                         break_frac=0.1, seed=2),
    "sentinel2": StackSpec(P=10980 * 10980, N=700, n_hist=350, miss=0.5, mask="iid",
                           f=73.0, year0=2016.0, break_frac=0.1, seed=4),
    # the Landsat scene with a complete history (the [27]
    # special case, L93); gaps (60% cloud) only in the monitoring period
    "dense": StackSpec(P=4096 * 4096, N=400, n_hist=200, miss=0.6, mask="cloud",
                       break_frac=0.1, seed=6, dense_hist=True),
    # a dated cube in which most slices hold no value at all
    # (Africa: ~350 of 6873 dates per image, L379): 2000 dates at 16 days
    # (f = 23), 88% of them empty, 50% i.i.d. gaps in the others
    "africa": StackSpec(P=1 << 23, N=2000, n_hist=1000, miss=0.5, mask="iid",
                        break_frac=0.1, seed=7, empty_frac=0.88),
}


def sweep_spec(N: int, miss: float, k: int, P: int = 4096 * 4096, index: int = 0) -> StackSpec:
    """configs[2]: N in {100,250,500,1000} x miss in {.1,.5,.9} x k in {1,3,5}."""
    return StackSpec(P=P, N=N, n_hist=N // 2, k=k, miss=miss, mask="iid",
                     break_frac=0.1, seed=100 + index)


def make_dates(N: int, f: float = 23.0, year0: float = 2000.0) -> np.ndarray:
    t = np.arange(1, N + 1, dtype=np.float64)
    return year0 + t / f


def _gen(device, seed: int, stream: int) -> torch.Generator:
    g = torch.Generator(device=device)
    g.manual_seed((int(seed) * 1_000_003 + int(stream) * 7919 + 12345) % (2**63 - 1))
    return g


def _grid_shape(P: int):
    W = int(math.isqrt(P))
    if W * W < P:
        W += 1
    H = (P + W - 1) // W
    return H, W


BLOCK = 1 << 20  # pixels per independently seeded block


def generate(spec: StackSpec, device="cpu", ldY: int | None = None, out: torch.Tensor | None = None,
             return_truth: bool = False, chunk_elems: int = 1 << 28, columns: tuple | None = None):
    """Return (Y [N][ldY] float32 on `device`, dates float64 numpy[, truth]).

    Block-deterministic: pixel parameters, noise and i.i.d. masks are drawn
    per block of BLOCK pixels from their own seeds, and the cloud field of a
    date from a global lattice, so `columns=(b, e)` generates exactly the
    pixels [b, e) of the full scene (a shard for strong scaling) without
    generating the rest.  Y then holds e - b columns."""
    P, N = int(spec.P), int(spec.N)
    b0, e0 = (0, P) if columns is None else (int(columns[0]), int(columns[1]))
    W_ = e0 - b0
    ldY = W_ if ldY is None else int(ldY)
    if ldY < W_:
        raise ValueError("ldY < number of columns")
    dev = torch.device(device)
    if out is None:
        Y = torch.empty((N, ldY), dtype=torch.float32, device=dev)
    else:
        Y = out
        assert Y.shape == (N, ldY) and Y.dtype == torch.float32
    dates = make_dates(N, spec.f, spec.year0)
    H, Wd = _grid_shape(P)
    two_pi = 2.0 * math.pi
    dd = torch.tensor(dates - dates[0], dtype=torch.float32, device=dev)
    sin_t = torch.tensor(np.stack([np.sin(two_pi * j * dates) for j in (1, 2, 3)]),
                         dtype=torch.float32, device=dev)
    cos_t = torch.tensor(np.stack([np.cos(two_pi * j * dates) for j in (1, 2, 3)]),
                         dtype=torch.float32, device=dev)
    cover = None
    if spec.mask == "cloud":
        gc0 = _gen(dev, spec.seed, 3)
        m = float(spec.miss)
        lo, hi = max(0.0, 2 * m - 1), min(1.0, 2 * m)
        cover = (torch.rand(N, generator=gc0, device=dev) * (hi - lo) + lo).cpu().numpy()
    truth = {"has_break": [], "delta": [], "t0": [], "noise_sd": []}
    tidx = torch.arange(N, device=dev)
    Tc = max(1, min(N, chunk_elems // max(min(W_, BLOCK), 1)))
    first_blk, last_blk = b0 // BLOCK, (e0 - 1) // BLOCK if e0 > b0 else b0 // BLOCK - 1
    for blk in range(first_blk, last_blk + 1):
        pb, pe = blk * BLOCK, min(P, (blk + 1) * BLOCK)   # block in scene coordinates
        sb, se = max(pb, b0), min(pe, e0)                # part of it we want
        nb = pe - pb
        g = _gen(dev, spec.seed, 1_000_000 + blk)
        u = lambda lo_, hi_, *shape: torch.rand(*shape, generator=g, device=dev) * (hi_ - lo_) + lo_
        a = u(0.3, 0.8, nb)
        b = u(-0.01, 0.01, nb)
        amp_s = u(-0.1, 0.1, 3, nb)
        amp_c = u(-0.1, 0.1, 3, nb)
        s = u(spec.noise_lo, spec.noise_hi, nb)
        has_break = torch.rand(nb, generator=g, device=dev) < spec.break_frac
        delta = u(0.1, 0.5, nb) * has_break
        t0 = torch.randint(spec.n_hist, N, (nb,), generator=g, device=dev)
        sl = slice(sb - pb, se - pb)
        if return_truth:
            truth["has_break"].append(has_break[sl]); truth["delta"].append(delta[sl])
            truth["t0"].append(t0[sl]); truth["noise_sd"].append(s[sl])
        for c0 in range(0, N, Tc):
            c1 = min(N, c0 + Tc)
            gcn = _gen(dev, spec.seed, 2_000_000 + blk * 65536 + c0)
            blkv = a[None, :] + b[None, :] * dd[c0:c1, None]
            for j in range(3):
                blkv += amp_s[j][None, :] * sin_t[j, c0:c1, None]
                blkv += amp_c[j][None, :] * cos_t[j, c0:c1, None]
            blkv += torch.randn(c1 - c0, nb, generator=gcn, device=dev) * s[None, :]
            blkv -= delta[None, :] * (tidx[c0:c1, None] >= t0[None, :])
            if spec.mask == "iid":
                miss = torch.rand(c1 - c0, nb, generator=gcn, device=dev) < spec.miss
                if spec.dense_hist:
                    miss[: max(0, min(c1, spec.n_hist) - c0)] = False
                blkv.masked_fill_(miss, float("nan"))
            elif spec.mask == "cloud":
                for t in range(max(c0, spec.n_hist) if spec.dense_hist else c0, c1):
                    field, thr = _cloud_rows(H, Wd, P, spec.seed, t, float(cover[t]), pb, pe, dev)
                    blkv[t - c0].masked_fill_(field < thr, float("nan"))
            elif spec.mask != "none":
                raise ValueError(spec.mask)
            if spec.empty_frac > 0:
                ge = _gen(dev, spec.seed, 4)
                empty = torch.rand(N, generator=ge, device=dev) < spec.empty_frac
                blkv[empty[c0:c1]] = float("nan")
            Y[c0:c1, sb - b0:se - b0] = blkv[:, sl]
            del blkv
    if ldY > W_:
        Y[:, W_:] = float("nan")
    if return_truth:
        truth = {k: torch.cat(v) for k, v in truth.items()}
        return Y, dates, truth
    return Y, dates


_FIELD_CACHE = {}


def _cloud_rows(H, W, P, seed, t, cover, pb, pe, dev):
    """Cloud field values for scene pixels [pb, pe) at date t, and the date's
    threshold (the cover-quantile of the full field, from a fixed subsample)."""
    key = (H, W, seed, t, str(dev))
    if key not in _FIELD_CACHE:
        if len(_FIELD_CACHE) > 8192:
            _FIELD_CACHE.clear()
        g = _gen(dev, seed, 3_000_000 + t)
        gh, gw = H // 64 + 2, W // 64 + 2
        lat = torch.rand(1, 1, gh, gw, generator=g, device=dev)
        # threshold from a coarse full-field sample (every 8th row / column)
        coarse = torch.nn.functional.interpolate(lat, size=((gh - 1) * 8 + 1, (gw - 1) * 8 + 1),
                                                 mode="bilinear", align_corners=True)
        thr = torch.quantile(coarse[0, 0, : (H + 7) // 8, : (W + 7) // 8].reshape(-1)[: 1 << 24], cover)
        _FIELD_CACHE[key] = (lat, thr)
    lat, thr = _FIELD_CACHE[key]
    gh, gw = lat.shape[2], lat.shape[3]
    r0, r1 = pb // W, (pe - 1) // W + 1
    # rows r0..r1-1 of the bilinear upsampling (align_corners: row y <-> lattice y/64)
    lr0, lr1 = r0 // 64, min(gh - 1, (r1 - 1) // 64 + 1)
    sub = lat[:, :, lr0:lr1 + 1, :]
    up = torch.nn.functional.interpolate(sub, size=((lr1 - lr0) * 64 + 1, (gw - 1) * 64 + 1),
                                         mode="bilinear", align_corners=True)[0, 0]
    rows = up[r0 - lr0 * 64: r1 - lr0 * 64, :W].reshape(-1)
    off = pb - r0 * W
    return rows[off: off + (pe - pb)], thr


def sample_columns(Y: torch.Tensor, P: int, count: int, seed: int = 0) -> np.ndarray:
    """Uniformly sampled pixel indices (sorted), for sampled parity/baselines."""
    rng = np.random.default_rng(seed)
    count = min(count, P)
    return np.sort(rng.choice(P, size=count, replace=False)).astype(np.int64)


def quantize_i16(Y: torch.Tensor, scale: float, offset: float, nodata: int = -32768) -> torch.Tensor:
    """Scaled int16 codes of a float stack (the NDMI product encoding of
    SURVEY 8(f) f4): code = round((y - offset) / scale) clipped to the int16
    range minus the nodata code, NaN -> nodata.  Input generation only."""
    lo, hi = -32768.0, 32767.0
    if nodata == -32768:
        lo = -32767.0
    elif nodata == 32767:
        hi = 32766.0
    codes = torch.empty(Y.shape, dtype=torch.int16, device=Y.device)
    for r in range(0, Y.shape[0], 16):  # row blocks: bounded fp64 temporaries
        y = Y[r:r + 16]
        q = torch.round((y.double() - offset) / scale).clamp(lo, hi)
        codes[r:r + 16] = torch.where(torch.isnan(y), torch.full_like(q, float(nodata)), q).to(torch.int16)
    return codes
