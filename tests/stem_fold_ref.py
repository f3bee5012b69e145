"""Test-side restatement of the stem fold (D16), written from its
formula, for the CPU identity test and the GPU workspace check.  Not product
code (the product's fold is the layout kernel, elementwise.cuh layout_fold)."""
import numpy as np


def fold_geometry(h, w, c, r, s, stride, pad):
    sh, sw = stride
    ph, pw = pad
    p = (h + 2 * ph - r) // sh + 1
    q = (w + 2 * pw - s) // sw + 1
    r2 = -(-r // sh)
    return p, q, r2, p + r2 - 1


def fold_input(x, r, s, stride, pad):
    """x [n, c, h, w] -> Y [n, 64, T, Q]:
    Y[n, j*s*c + sx*c + ci, t, q] = x[n, ci, sh*t - ph + j, sw*q - pw + sx] (0 outside)."""
    n, c, h, w = x.shape
    sh, sw = stride
    ph, pw = pad
    p, q, r2, t_rows = fold_geometry(h, w, c, r, s, stride, pad)
    y = np.zeros((n, 64, t_rows, q))
    for j in range(sh):
        for sx in range(s):
            for ci in range(c):
                cc = j * s * c + sx * c + ci
                for t in range(t_rows):
                    hh = sh * t - ph + j
                    if not 0 <= hh < h:
                        continue
                    for qq in range(q):
                        ww = sw * qq - pw + sx
                        if 0 <= ww < w:
                            y[:, cc, t, qq] = x[:, ci, hh, ww]
    return y


def fold_weights(wt, stride):
    """wt [k, c, r, s] -> W' [k, 64, R2, 1]:
    W'[k, j*s*c + sx*c + ci, r2] = wt[k, ci, sh*r2 + j, sx] (0 where sh*r2 + j >= r)."""
    k, c, r, s = wt.shape
    sh = stride[0]
    r2n = -(-r // sh)
    out = np.zeros((k, 64, r2n, 1))
    for j in range(sh):
        for sx in range(s):
            for ci in range(c):
                cc = j * s * c + sx * c + ci
                for r2 in range(r2n):
                    if sh * r2 + j < r:
                        out[:, cc, r2, 0] = wt[:, ci, sh * r2 + j, sx]
    return out
