/*
 * tcgen.h — seeded synthetic edge-list generators (C ABI).
 *
 * These generators are the ONLY code shared by the CUDA path and the CPU
 * oracle: they produce inputs, never counts.  They hold none of the triangle
 * counting arithmetic (no dedup, orientation or intersection) — an edge list
 * they emit may contain self-loops and duplicate / reversed pairs, exactly
 * like the raw SNAP files the paper cleans (§IV "Datasets").
 *
 * Randomness is counter based: every random word is
 * splitmix64(f(seed, stream, counter)), and every probabilistic decision is an
 * INTEGER comparison against a 32-bit threshold floor(p * 2^32), so the output
 * is a pure function of the arguments (independent of thread count).
 *
 * Shapes follow SURVEY.md §8(d): RMAT/Kronecker (Graph500 initiator,
 * configs C1/C3/C4), Chung-Lu power law shaped like com-LiveJournal (C2,
 * PAPER.md Table II), and a road-like triangulated lattice (C5, shaped
 * like RoadNet-CA, Table II).
 *
 * Ownership: the caller allocates src/dst (host memory, int32) of the size
 * stated per function; nothing is allocated that outlives a call.
 * Errors: a negative return value is an error (bad argument); no abort.
 */
#ifndef TCGEN_H
#define TCGEN_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* Number of worker threads the generators use (0 = hardware_concurrency). */
void tcgen_set_threads(int threads);

/*
 * RMAT (Chakrabarti et al.; Graph500 Kronecker generator without noise).
 * Emits exactly edge_factor << scale pairs into src/dst (pair i is a pure
 * function of (seed, i)).  thr_a, thr_ab, thr_abc are the cumulative
 * quadrant thresholds as 32-bit fixed point: quadrant 0 if r < thr_a,
 * 1 if r < thr_ab, 2 if r < thr_abc, else 3 (r = 32 random bits per level).
 * Graph500 (0.57, 0.19, 0.19, 0.05) is thr = (2448131358, 3264175144,
 * 4080218930).  permute != 0 applies a seeded bijection of [0, 2^scale) to
 * every label (Graph500 vertex scrambling).  Vertex ids are < 2^scale.
 * Returns the number of pairs written, or -1 on bad arguments
 * (scale outside [1, 31], edge_factor < 1).
 */
int64_t tcgen_rmat(uint64_t seed, int scale, int64_t edge_factor,
                   uint32_t thr_a, uint32_t thr_ab, uint32_t thr_abc,
                   int permute, int32_t* src, int32_t* dst);

/*
 * Chung-Lu power-law graph: num_pairs endpoint pairs, each endpoint drawn
 * i.i.d. with probability proportional to w_i = min(w_max, c * (i+1)^(-1/(gamma-1))),
 * c chosen so that sum(w) = 2 * num_pairs.  Sampling is by upper_bound of a
 * 64-bit random word in a 64-bit fixed-point CDF.  Vertex ids are < n.
 * Returns num_pairs, or -1 on bad arguments.
 */
int64_t tcgen_chung_lu(uint64_t seed, int64_t n, int64_t num_pairs, double gamma,
                       double w_max, int32_t* src, int32_t* dst);

/*
 * Road-like lattice: side x side grid, vertex (r, c) = r * side + c.  Each of
 * the 2*side*(side-1) grid edges is kept when a random word < thr_keep, and
 * the diagonal (r,c)-(r+1,c+1) of each of the (side-1)^2 cells is kept when a
 * random word < thr_diag.  Writes at most tcgen_lattice_capacity(side) pairs
 * (the caller's buffer size) and returns the number written, -1 on error.
 */
int64_t tcgen_lattice_capacity(int64_t side);
int64_t tcgen_lattice(uint64_t seed, int64_t side, uint32_t thr_keep, uint32_t thr_diag,
                      int32_t* src, int32_t* dst);

/* FNV-style order-sensitive checksum of an edge list (host), for reproducibility pins. */
uint64_t tcgen_checksum(const int32_t* src, const int32_t* dst, int64_t num_pairs);

#ifdef __cplusplus
}
#endif
#endif /* TCGEN_H */
