"""CPU oracle for the mixed-precision Matérn log-likelihood path — TEST INFRASTRUCTURE ONLY.

Plain, slow, obviously-correct FP64 implementation of what the GPU hot path
computes, written from the paper (Cao et al., IEEE CLUSTER 2023,
/root/reference/PAPER.md, cited as P:<line>) and nothing else.

Who may use it: only `tests/`, `__graft_entry__.smoke()` and the `cpu_baseline`
/ `--impl reference` legs of `bench.py`.  The product package
(`paper_conf_cluster_caoalgkb23_b200`) never imports it, and it never imports
the product package: the two share no code.  The only shared module is
`synth` (seeded input recipes, no method arithmetic).

Modules (each function cites the passage it follows):
  matern     — 2D Matérn covariance C(h; theta)                     P:82  §III-A
  tiles      — tiling, tile generation, tile Frobenius norms       P:117 §V
  precision  — kernel / storage / communication precision maps     P:117, Alg. 2
  cholesky   — right-looking tile Cholesky (Alg. 1), FP64; optional
               mixed-precision emulation following the maps
  loglik     — Eq. (1): log-determinant, forward solve, l(theta)

Pins (what fixes each part independently of this code; tests/test_oracle_*.py):
  matern     — closed forms nu = 1/2, 3/2, 5/2; mpmath.besselk at 40 digits;
               C(0) = sigma^2; monotone decay in h.                         pinned
  tiles      — tile_sqnorm / global_sqnorm against the dense ||A||_F^2 of the
               whole symmetric matrix and against hand-derived closed forms of
               the Kac-Murdock-Szego matrix per tile; correct rounding on
               hand-built sums (test_oracle_pins.py).                       pinned
  cholesky / loglik — Kac-Murdock-Szego closed forms (L, log|Sigma|, Z^T Sigma^-1 Z);
               mpmath 50-digit determinant and solve at n = 40;
               tile factor vs dense LAPACK; non-SPD `info`.                  pinned
  residual   — hand-computed 2 x 2 example (both triangles of A).           pinned
  precision (kernel/storage map) — hand-built norm arrays with known
               answers (ties at both thresholds), one tile on each side of
               each threshold, literal storage table, monotonicity.          pinned
  precision (band map, reading C21) — hand-built norms with a known band,
               both too-narrow and too-wide checked.                         pinned
  precision (comm map, Alg. 2) — text claims: all-FP64 map -> comm FP64;
               extreme FP64/FP16 map -> every communication STC;
               hand-built successor cases.  The paper's Fig. 4b example is
               an image (absent): that example is parity unpinned.          partially pinned
  cholesky MP-emulation mode — predicts the MP error only and is NOT a pass
               criterion anywhere: the MP tests compare the GPU with the FP64
               definition (north-star tolerance) and with a backward-error
               bound computed from the maps.                                parity unpinned (emulation)
"""

FP64, FP32, FP16 = 0, 1, 2  # smaller value = higher precision (SURVEY §8(b) mp_prec)
FP16H = 3  # four-level maps only: the paper's pure FP16 class (FP16 operands AND accumulation)
PREC_NAMES = {FP64: "FP64", FP32: "FP32", FP16: "FP16_32", FP16H: "FP16"}
