"""Pins for the full-size certificates of tests/props.py: on seeded small graphs the
oracle's rows pass them, and single-element corruptions of a row (a value off by one,
a wrong pred / succ id, an unreached vertex marked reached) are caught."""
import numpy as np
import pytest
import torch

import oracle
import tgsynth
from tests import props

NONE = 0xFFFFFFFF


def _t(a):
    return torch.from_numpy(np.ascontiguousarray(a, np.uint32).view(np.int32))


def _graph(seed):
    ge = tgsynth.make_graph("C1", device="cpu", scale_shift=-6)  # 256 vertices, 4096 edges
    n, u, v, t, d, w = ge.numpy()
    return n, u, v, t, d


@pytest.mark.parametrize("win", [(0, 0x7FFFFFFE), (250, 750)])
def test_oracle_rows_pass(win):
    n, u, v, t, d = _graph(0)
    og = oracle.Graph(n, u, v, t, d)
    for x in (0, 1, 7):
        A, P, _ = oracle.eat(og, x, *win)
        props.check_eat_row(_t(u), _t(v), _t(t), _t(d), n, x, win, _t(A), _t(P), chunk=1000)
        L, S, _ = oracle.ld(og, x, *win)
        props.check_ld_row(_t(u), _t(v), _t(t), _t(d), n, x, win, _t(L), _t(S), chunk=1000)


def _corruptions(vals, ids, x, rng):
    """single-element corruptions of a row: value +-1, id changed, unreached -> reached"""
    reached = [i for i in range(len(vals)) if vals[i] != NONE and i != x]
    unreached = [i for i in range(len(vals)) if vals[i] == NONE]
    out = []
    for i in rng.choice(reached, size=min(6, len(reached)), replace=False):
        a = vals.copy(); a[i] += 1; out.append((a, ids))
        a = vals.copy(); a[i] -= 1; out.append((a, ids))
        b = ids.copy(); b[i] = (b[i] + 1) % 4096; out.append((vals, b))
    for i in unreached[:3]:
        a = vals.copy(); a[i] = 500; out.append((a, ids))
    return out


def test_corruptions_caught():
    n, u, v, t, d = _graph(0)
    og = oracle.Graph(n, u, v, t, d)
    rng = np.random.default_rng(5)
    win = (0, 0x7FFFFFFE)
    args = (_t(u), _t(v), _t(t), _t(d), n)
    A, P, _ = oracle.eat(og, 0, *win)
    for a, p in _corruptions(A, P, 0, rng):
        with pytest.raises(AssertionError):
            props.check_eat_row(*args, 0, win, _t(a), _t(p), chunk=1000)
    L, S, _ = oracle.ld(og, 0, *win)
    for a, p in _corruptions(L, S, 0, rng):
        with pytest.raises(AssertionError):
            props.check_ld_row(*args, 0, win, _t(a), _t(p), chunk=1000)
