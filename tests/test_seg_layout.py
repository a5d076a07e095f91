"""Host-side checks of the row-segment layout helpers of the CUDA path
(csrc/clover_common.cuh), compiled by nvcc as host code -- no GPU needed.

seg_rows_lay maps a kernel's launch slots to row segments.  In the band
layout the rows are cut into ch bands walked wave-major:
every row must be covered exactly once, each band's segments must follow
each other in launch order, and each band must end in its half-height tail
segments; the row layout (ch = 0) must tile the rows as before."""
from __future__ import annotations

import os
import shutil
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CSRC = os.path.join(ROOT, "paper_conf_cluster_regulymg15_b200", "csrc")

PROG = r"""
#include "clover_common.cuh"
#include <cstdio>
#include <vector>
using namespace clover;
static int fail(const char* what, int ks, int rows, int ch, int s) {
  printf("FAIL %s ks=%d rows=%d ch=%d s=%d\n", what, ks, rows, ch, s);
  return 1;
}
int main() {
  long banded = 0;
  // band layout: every row covered exactly once by the non-empty segments;
  // within a band the segments ascend with the launch slot (consecutive
  // rows), the band's first segment is in wave 0 and its last
  // CLOVER_TAIL_WAVES segments have ks / CLOVER_TAIL_DIV rows
  for (int td = 2; td <= 4; td += 2)
  for (int ks = 8; ks <= 64; ks *= 2)
    for (int rows = 1; rows <= 4200; rows += (rows < 300 ? 1 : 97))
      for (int C = 0; C <= 40; ++C) {
        int ch, cf;
        band_params(ks, C, rows, &ch, &cf, td);
        if (ch == 0) continue;
        ++banded;
        const int n = seg_count_lay(ks, 0, ch, cf, rows, td);
        if (n != (cf + CLOVER_TAIL_WAVES) * ch) return fail("count", ks, rows, ch, n);
        std::vector<int> cover(rows + 2, 0);
        for (int c = 0; c < ch; ++c) {
          int next = -1;
          for (int w = 0; w < cf + CLOVER_TAIL_WAVES; ++w) {
            const int s = w * ch + c;
            int k0, len;
            seg_rows_lay(s, ks, 0, ch, cf, rows, k0, len, td);
            if (len > ks) return fail("len", ks, rows, ch, s);
            if (w >= cf && len != ks / td) return fail("tail", ks, rows, ch, s);
            if (len <= 0) continue;
            if (next >= 0 && k0 != next) return fail("band order", ks, rows, ch, s);
            next = k0 + len;
            for (int k = k0; k < k0 + len; ++k) {
              if (k < 1 || k > rows) return fail("range", ks, rows, ch, s);
              cover[k]++;
            }
          }
        }
        for (int k = 1; k <= rows; ++k)
          if (cover[k] != 1) return fail("cover", ks, rows, ch, k);
      }
  // row layout (ch = 0): full segments then half-height tail segments
  for (int td = 2; td <= 4; td += 2)
  for (int ks = 16; ks <= 64; ks *= 2)
    for (int nb = 0; nb <= 40; ++nb)
      for (int rows = 1; rows <= 2000; rows += 37) {
        const int n = seg_count_lay(ks, nb, 0, 0, rows, td);
        int next = 1;
        for (int s = 0; s < n; ++s) {
          int k0, len;
          seg_rows_lay(s, ks, nb, 0, 0, rows, k0, len, td);
          if (k0 != next || len <= 0) return fail("rows", ks, rows, nb, s);
          next = k0 + len;
        }
        if (next <= rows || next - rows > ks) return fail("row cover", ks, rows, nb, n);
      }
  printf("ok %ld\n", banded);
  return 0;
}
"""


def _nvcc():
    for c in (os.environ.get("NVCC"), "/usr/local/cuda/bin/nvcc", shutil.which("nvcc")):
        if c and os.path.exists(c):
            return c
    return None


@pytest.mark.skipif(_nvcc() is None, reason="nvcc not available")
def test_band_and_row_layouts_tile_the_rows(tmp_path):
    src = tmp_path / "seg.cu"
    src.write_text(PROG)
    exe = tmp_path / "seg"
    subprocess.check_call([_nvcc(), "-std=c++17", "-O1", "-I", CSRC, "-o", str(exe), str(src)],
                          cwd=tmp_path)
    out = subprocess.run([str(exe)], capture_output=True, text=True)
    assert out.returncode == 0, out.stdout + out.stderr
    assert out.stdout.startswith("ok"), out.stdout
