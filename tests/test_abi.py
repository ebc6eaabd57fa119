"""The C-ABI library without a GPU: it loads, exports every symbol that
include/eim.h declares, and its host-only logic (IMM parameters, shard
ranges, argument validation) is right.  No compute calls."""
import ctypes
import os
import re

import numpy as np
import pytest

import oracle
import paper_conf_sc_doneyhl25_b200 as eim
from paper_conf_sc_doneyhl25_b200 import _build

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module", autouse=True)
def built():
    _build.build()


def _declared():
    src = open(os.path.join(ROOT, "include", "eim.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(eim_[a-z0-9_]+)\s*\(", src)))


def test_header_symbols_exported():
    declared = _declared()
    assert len(declared) >= 12
    L = ctypes.CDLL(eim.LIB_PATH)
    for name in declared:
        assert hasattr(L, name), name
    assert sorted(eim.EXPORTS) == declared


def test_version_and_no_gpu_error_path():
    assert "sm_100a" in eim.eim_version()
    if not _has_gpu():
        with pytest.raises(eim.EimError) as ei:
            eim.eim_create(0)
        assert ei.value.status == eim.EIM_E_CUDA
        assert eim.eim_last_error(None)


def _has_gpu():
    try:
        import torch
        return torch.cuda.is_available()
    except Exception:
        return False


def test_invalid_create_arguments():
    for args in [(-1, 0, 1), (0, 1, 1), (0, 0, 0), (0, 0, 2)]:
        with pytest.raises(eim.EimError) as ei:
            eim.eim_create(*args)
        assert ei.value.status == eim.EIM_E_INVAL


@pytest.mark.parametrize("n,k,eps,ell", [(1024, 5, 0.5, 1.0), (4847571, 50, 0.5, 1.0), (3072441, 100, 0.3, 1.0),
                                         (41652230, 50, 0.5, 1.0), (65608366, 200, 0.1, 1.0), (2, 2, 0.01, 3.0)])
def test_imm_params_bit_identical_to_oracle(n, k, eps, ell):
    a = eim.eim_imm_params(n, k, eps, ell)
    b = oracle.imm_params(n, k, eps, ell)
    for f in ("ell_p", "eps_p", "lnC", "lambda_p", "lambda_s", "log2n"):
        assert getattr(a, f) == getattr(b, f), f


def test_imm_params_validation():
    for args in [(1, 1, 0.5, 1.0), (10, 0, 0.5, 1.0), (10, 11, 0.5, 1.0), (10, 1, 1.0, 1.0), (10, 1, 0.5, -1.0)]:
        with pytest.raises(eim.EimError) as ei:
            eim.eim_imm_params(*args)
        assert ei.value.status == eim.EIM_E_INVAL


@pytest.mark.parametrize("first,count,world", [(0, 0, 1), (0, 10, 3), (7, 101294, 8), (2**40, 12345, 5), (3, 2, 4)])
def test_shard_ranges_partition(first, count, world):
    pieces = [eim.eim_shard_range(first, count, r, world) for r in range(world)]
    assert pieces[0][0] == first and pieces[-1][1] == first + count
    for (a, b), (c, d) in zip(pieces, pieces[1:]):
        assert b == c and a <= b
    sizes = [b - a for a, b in pieces]
    assert max(sizes) - min(sizes) <= 1
    with pytest.raises(eim.EimError):
        eim.eim_shard_range(0, 10, world, world)


def test_create_group_argument_checks():
    for devs in ([], [-1], [0, -2]):
        with pytest.raises(eim.EimError) as ei:
            eim.eim_create_group(devs)
        assert ei.value.status == eim.EIM_E_INVAL
    if not _has_gpu():
        with pytest.raises(eim.EimError) as ei:
            eim.eim_create_group([0, 0])
        assert ei.value.status == eim.EIM_E_CUDA
