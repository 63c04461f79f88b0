"""GPU parity of bcf_set_op_u32 (merge-path set operations on the CF merge,
PAPER.md:380) against the oracle (oracle/setops_oracle.c, ISO C++ multiset
semantics), keys and source tags, bit-exact: sizes across many merge tiles
and compaction blocks, ragged tails, empty sides, duplicate-heavy keys with
runs spanning blocks, identical and disjoint inputs."""
import numpy as np
import pytest

import oracle
import synthetic_inputs as si

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

import paper_conf_spaa_berneys25_b200 as bcf  # noqa: E402

if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("no CUDA device", allow_module_level=True)

DEV = torch.device("cuda:0")
OPS = ["union", "intersection", "difference", "symmetric_difference"]


def _dev(x):
    return torch.from_numpy(np.ascontiguousarray(x, dtype=np.uint32).view(np.int32).copy()).to(DEV)


def _check(op, a, b):
    k, s = bcf.set_op(op, _dev(a), _dev(b), with_source=True)
    ek, es = oracle.set_op_u32(op, a, b)
    np.testing.assert_array_equal(k.cpu().numpy().view(np.uint32), ek)
    np.testing.assert_array_equal(s.cpu().numpy().view(np.uint32), es)
    k2 = bcf.set_op(op, _dev(a), _dev(b))
    np.testing.assert_array_equal(k2.cpu().numpy().view(np.uint32), ek)


@pytest.mark.parametrize("op", OPS)
@pytest.mark.parametrize("na,nb", [(0, 0), (0, 17), (33, 0), (1, 1), (1000, 999), (4096, 4096), (100003, 77777),
                                   (3968 * 5 + 3, 4095)])
@pytest.mark.parametrize("mask", [0x3, 0xFFF, 0xFFFFFFFF])
def test_set_ops_match_oracle(op, na, nb, mask):
    seed = si.config_seed(8) + na * 7 + nb + mask % 97
    a = np.sort(si.uniform_u32(na, seed) & np.uint32(mask))
    b = np.sort(si.uniform_u32(nb, seed + 1) & np.uint32(mask))
    _check(op, a, b)


@pytest.mark.parametrize("op", OPS)
def test_set_ops_structured(op):
    x = np.sort(si.uniform_u32(50000, 3) & np.uint32(0xFFFF))
    _check(op, x, x)                                      # identical
    _check(op, np.arange(1000, dtype=np.uint32), np.arange(1000, 3000, dtype=np.uint32))   # disjoint
    _check(op, np.zeros(20000, np.uint32), np.zeros(30000, np.uint32))                      # one run of 50000
    _check(op, np.full(5, 0xFFFFFFFF, np.uint32), np.array([0, 0xFFFFFFFF], np.uint32))     # extremes


@pytest.mark.parametrize("op", OPS)
def test_set_ops_large(op):
    n = 1 << 22
    a = np.sort(si.uniform_u32(n, 11) & np.uint32(0xFFFFF))
    b = np.sort(si.uniform_u32(n - 12345, 12) & np.uint32(0xFFFFF))
    _check(op, a, b)
