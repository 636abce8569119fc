"""An independent float64 evaluation of the pipeline, used ONLY to pin the oracle.

It is written differently from oracle/oracle.c on purpose, so that a slip in
one is not repeated in the other:
  * downscale by numpy reshape-sum;
  * body upscale as half-pixel-centre bilinear interpolation of D
    (scipy RegularGridInterpolator) -- the closed form that the 4x2
    parameter matrix P of Fig. 5 (R3) implements;
  * border upscale from a per-pixel FINAL-STATE rule derived by hand from the
    step order of L140-L142 (the oracle executes the steps in sequence);
  * Sobel with scipy.ndimage.sobel, 3x3 min/max with scipy filters;
  * the strength / oscStrength factors and the overshoot chain in float64
    with NO float32 rounding anywhere (the "exact" real-number result).
Nothing here imports the oracle or the CUDA package.
"""
import numpy as np
from scipy import ndimage
from scipy.interpolate import RegularGridInterpolator


def downscale(O):
    H, W = O.shape
    return O.astype(np.int64).reshape(H // 4, 4, W // 4, 4).sum(axis=(1, 3)) / 16.0


def body_bilinear(D, H, W):
    """U on rows/cols 2..H-3 / 2..W-3: bilinear in D sampled at pixel centres.
    Block i of D covers pixels 4i..4i+3, whose centre is 4i+1.5."""
    h, w = D.shape
    f = RegularGridInterpolator((4 * np.arange(h) + 1.5, 4 * np.arange(w) + 1.5), D)
    rr, cc = np.meshgrid(np.arange(2, H - 2), np.arange(2, W - 2), indexing="ij")
    return f(np.stack([rr.ravel(), cc.ravel()], axis=1)).reshape(rr.shape)


def border_rule(D, H, W):
    """Final value of every pixel of the 2-pixel border ring (NaN elsewhere).

    Derived from L140-L142 by asking, for each pixel, which step writes it
    LAST: (vii) bottom-right 2x2; (vi) columns 1 and W-1 copy columns 0 and
    W-2 on rows 0..H-3; (v) rows 1 and H-1 copy rows 0 and H-2 on columns
    0..W-3; (i)-(iv) the four line passes."""
    h, w = D.shape

    def rowline(i, c):  # line(D[i, :], W)[c], c in [0, W-3]
        if c == W - 3:
            c = W - 4
        j, k = divmod(c, 4)
        return D[i, j] if k == 0 else ((4 - k) * D[i, j] + k * D[i, j + 1]) / 4

    def colline(j, r):  # line(D[:, j], H)[r], r in [0, H-3]
        if r == H - 3:
            r = H - 4
        i, k = divmod(r, 4)
        return D[i, j] if k == 0 else ((4 - k) * D[i, j] + k * D[i + 1, j]) / 4

    U = np.full((H, W), np.nan)
    for r in range(H):
        for c in range(W):
            if not (r <= 1 or r >= H - 2 or c <= 1 or c >= W - 2):
                continue
            if r >= H - 2 and c >= W - 2:
                U[r, c] = colline(w - 1, H - 3)
            elif c <= 1 and r <= H - 3:
                U[r, c] = D[0, 0] if r <= 1 else colline(0, r)
            elif c >= W - 2 and r <= H - 3:
                U[r, c] = colline(w - 1, r)
            elif r <= 1:
                U[r, c] = rowline(0, c)
            else:
                U[r, c] = rowline(h - 1, c)
    return U


def upscale(O):
    H, W = O.shape
    D = downscale(O)
    U = border_rule(D, H, W)
    U[2:H - 2, 2:W - 2] = body_bilinear(D, H, W)
    return U


def sobel(O):
    o = O.astype(np.float64)
    gx = ndimage.sobel(o, axis=1, mode="constant")
    gy = ndimage.sobel(o, axis=0, mode="constant")
    pE = (np.abs(gx) + np.abs(gy)).astype(np.int64)
    pE[0, :] = pE[-1, :] = 0
    pE[:, 0] = pE[:, -1] = 0
    return pE


def sharpen_f64(O, amount, gamma, osc_gain, osc_scale):
    """Real-number (float64, no f32 rounding) result F before the 8-bit
    rounding, plus S."""
    H, W = O.shape
    o = O.astype(np.float64)
    U = upscale(O)
    E = o - U
    pE = sobel(O)
    S = int(pE.sum())
    m = max(S / (W * H), 1.0)
    with np.errstate(divide="ignore"):
        adj = amount * np.power(pE / m, gamma)
    if gamma == 0:
        adj = np.full(pE.shape, float(amount))
    P = adj * E + U
    mx = ndimage.maximum_filter(o, size=3, mode="nearest")
    mn = ndimage.minimum_filter(o, size=3, mode="nearest")
    osc = np.clip(osc_gain * np.exp(-pE / (osc_scale * m)), 0, 1)
    F = np.where(P > mx, np.minimum(mx + osc * (P - mx), 255),
                 np.where(P < mn, np.maximum(mn + osc * (P - mn), 0), np.clip(P, 0, 255)))
    frame = np.zeros((H, W), bool)
    frame[0, :] = frame[-1, :] = frame[:, 0] = frame[:, -1] = True
    F[frame] = np.clip(P[frame], 0, 255)
    return F, S
