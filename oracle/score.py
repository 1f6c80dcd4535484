"""Discriminant scoring (TEST INFRASTRUCTURE ONLY).

P:175  z = W_out h_T^(L)                    (only the N identifier rows are needed)
P:179  s_i = exp(z[v_i]) / sum_j exp(z[v_j])
P:183  TopK_{i in [1,N]} s_i                (ties -> lower candidate index, reading R9b)
"""
from __future__ import annotations

import numpy as np


def softmax(z: np.ndarray) -> np.ndarray:
    z = np.asarray(z, dtype=np.float64)
    e = np.exp(z - np.max(z))
    return e / np.sum(e)


def topk(s: np.ndarray, k: int) -> np.ndarray:
    """Indices of the k largest scores, descending; equal scores keep the lower index first."""
    s = np.asarray(s)
    order = sorted(range(len(s)), key=lambda i: (-s[i], i))
    return np.array(order[:k], dtype=np.int64)


def score(w_out_rows: np.ndarray, hf: np.ndarray, k: int = 0):
    """(z, s, topk) for identifier rows W_out[v_i] (N x H) and the final-normed hidden hf."""
    z = np.asarray(w_out_rows, dtype=np.float64) @ np.asarray(hf, dtype=np.float64)
    s = softmax(z)
    return z, s, topk(s, k) if k else np.zeros(0, dtype=np.int64)
