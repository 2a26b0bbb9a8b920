"""Pins for the oracle's random stream (R1, R2).

* Philox4x32-10 against the Random123 known-answer vectors (tests/golden/philox4x32_10_kat.txt).
* Philox4x32-10 against cuRAND's independent implementation (curand_philox4x32_x.h, compiled for the
  host with nvcc) on 20 000 random (counter, key) pairs.
* uniform(r, m) = floor(r m / 2^32): closed forms for powers of two and exact equidistribution.
* draw(seed, v, h, i) picks word i & 3 of the block with counter (lo v, hi v, h, i >> 2).
"""
import os
import shutil
import subprocess

import numpy as np
import pytest

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "philox4x32_10_kat.txt")


def _kat():
    rows = []
    for line in open(GOLDEN):
        if line.startswith("#") or not line.strip():
            continue
        w = [int(x, 16) for x in line.split()]
        rows.append((w[0:4], w[4:6], w[6:10]))
    return rows


def test_philox_known_answers(orc):
    rows = _kat()
    assert len(rows) == 3
    for ctr, key, want in rows:
        got = orc.philox4x32_10(ctr, key)
        assert [int(x) for x in got] == want


CURAND_SRC = r"""
#define QUALIFIERS static inline __host__ __device__
#include <curand_philox4x32_x.h>
#include <cstdio>
int main() {
  unsigned a[6];
  while (scanf("%u %u %u %u %u %u", &a[0], &a[1], &a[2], &a[3], &a[4], &a[5]) == 6) {
    uint4 c = {a[0], a[1], a[2], a[3]}; uint2 k = {a[4], a[5]};
    uint4 r = curand_Philox4x32_10(c, k);
    printf("%u %u %u %u\n", r.x, r.y, r.z, r.w);
  }
}
"""


@pytest.mark.skipif(shutil.which("nvcc") is None, reason="nvcc not available")
def test_philox_matches_curand(orc, tmp_path):
    src = tmp_path / "p.cu"
    src.write_text(CURAND_SRC)
    exe = tmp_path / "p"
    subprocess.run(["nvcc", "-Wno-deprecated-gpu-targets", "-o", str(exe), str(src)], check=True)
    rng = np.random.default_rng(123)
    vals = rng.integers(0, 2**32, size=(20000, 6), dtype=np.uint64)
    vals[:10] = 0
    vals[10:20] = 2**32 - 1
    inp = "\n".join(" ".join(str(int(x)) for x in row) for row in vals)
    out = subprocess.run([str(exe)], input=inp, capture_output=True, text=True, check=True).stdout.split("\n")
    for row, line in zip(vals, out):
        want = [int(x) for x in line.split()]
        got = [int(x) for x in orc.philox4x32_10(row[:4], row[4:])]
        assert got == want


def test_uniform_closed_forms(orc):
    rng = np.random.default_rng(5)
    for r in [0, 1, 2**31, 2**32 - 1] + [int(x) for x in rng.integers(0, 2**32, 200)]:
        for p in range(0, 33):
            # m = 2^p: floor(r 2^p / 2^32) = r >> (32 - p)
            assert orc.uniform(r, 2**p) == (r >> (32 - p) if p < 32 else r)
        assert orc.uniform(r, 1) == 0
        for m in [3, 7, 1000, 2**31 + 11]:
            u = orc.uniform(r, m)
            assert 0 <= u < m
    # extremes: the largest r maps to m-1, the smallest to 0
    for m in [2, 3, 5, 12345, 2**32 - 1]:
        assert orc.uniform(2**32 - 1, m) == m - 1
        assert orc.uniform(0, m) == 0


def test_uniform_equidistribution_exact(orc):
    # For m dividing 2^32 every output value has exactly 2^32/m preimages; check the preimage
    # boundaries r = c * 2^32 / m exactly (uniform jumps from c-1 to c there).
    for m in [2, 4, 64, 1024]:
        step = 2**32 // m
        for c in range(1, m, max(1, m // 16)):
            assert orc.uniform(c * step - 1, m) == c - 1
            assert orc.uniform(c * step, m) == c


def test_draw_word_selection(orc):
    seed = 0x0123456789ABCDEF
    v, h = 0x1_0000_0005, 2
    for i in range(12):
        block = orc.philox4x32_10([v & 0xFFFFFFFF, v >> 32, h, i >> 2], [seed & 0xFFFFFFFF, seed >> 32])
        assert orc.draw(seed, v, h, i) == int(block[i & 3])
