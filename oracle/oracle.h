/*
 * oracle.h -- CPU ORACLE for the GNNLab sample+extract hot path.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and
 * bench.py (its cpu_baseline leg and `--impl reference`) may load or call
 * anything under oracle/.  It shares no code, header, table or helper with
 * the CUDA library (paper_conf_eurosys_yangtswycyz22_b200/csrc); neither
 * includes the other.
 *
 * Plain, single-threaded, sequential C.  Every function follows the
 * definition it cites, in the paper's order:
 *   PAPER.md = /root/reference/PAPER.md (GNNLab, EuroSys'22),
 *   readings Q1..Q18 = SURVEY.md §8(c) / DESIGN.md "Readings".
 */
#ifndef GNNLAB_ORACLE_H
#define GNNLAB_ORACLE_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

enum { ORC_SHUFFLE = 1, ORC_KHOP = 2, ORC_RWALK = 3 };
enum { ORC_OK = 0, ORC_EINVAL = -1, ORC_ENOMEM = -2, ORC_ERANGE = -5 };

/* Philox4x32-10 (Random123).  out may alias ctr. */
void orc_philox(const uint32_t ctr[4], const uint32_t key[2], uint32_t out[4]);
/* c3 = (epoch & 0xFFFF) << 16 | (hop & 0xFF) << 8 | domain   (reading Q4) */
uint32_t orc_c3(uint32_t epoch, uint32_t hop, uint32_t domain);
/* draw64 = w1<<32|w0 (half 0) or w3<<32|w2 (half 1) of philox(ctr, key=(lo,hi)(seed)) */
uint64_t orc_draw64(uint64_t seed, uint32_t c0, uint32_t c1, uint32_t c2, uint32_t c3, int half);
/* floor(r * n / 2^64): uniform on [0,n) up to bias n/2^64 */
uint32_t orc_bounded(uint64_t r, uint32_t n);

/* Epoch shuffle (§6.2 "shuffle the training set T at the
 * beginning of each epoch"): out[j] = T[i_j] where i_j orders
 * (draw64(i,0,0,c3(epoch,0,SHUFFLE),0), i) ascending. */
int orc_shuffle(const uint32_t* T, uint64_t n, uint64_t seed, uint32_t epoch, uint32_t* out);

/* k-hop uniform neighbourhood sampling + dedup/relabel into per-hop blocks
 * (§2, Fig 7 L169-185, L230 Fig 9, L250 §5.2; readings Q1-Q7).
 *   lid_scratch: int32[V], every entry -1 on entry; restored to -1 on exit.
 *   uniq: gid by lid (cap uniq_cap); sizes[0..L] = n_0..n_L.
 *   blk_indptr: concatenation over hops of u32[n_l+1]; blk_indices: of
 *   u32[nnz_l] src lids; nnz[0..L-1].
 *   picks (nullable): concatenation over hops of u32[n_l * k_l] CSR
 *   positions chosen, 0xFFFFFFFF padded (diagnostic only). */
int orc_sample_khop(const uint64_t* indptr, const uint32_t* indices, uint64_t V,
                    const uint32_t* seeds, uint64_t n0, const uint32_t* fanouts, uint32_t L,
                    uint64_t seed, uint32_t epoch, uint32_t batch, int32_t* lid_scratch,
                    uint32_t* uniq, uint64_t uniq_cap, uint64_t* sizes,
                    uint32_t* blk_indptr, uint64_t indptr_cap,
                    uint32_t* blk_indices, uint64_t indices_cap, uint64_t* nnz,
                    uint32_t* picks, uint64_t picks_cap);

/* k-hop WEIGHTED sampling with replacement by inverse CDF over the row's edge
 * weights (L81, L148 fn5; reading Q19); weights: u32[E]. */
int orc_sample_khop_weighted(const uint64_t* indptr, const uint32_t* indices,
                             const uint32_t* weights, uint64_t V, const uint32_t* seeds,
                             uint64_t n0, const uint32_t* fanouts, uint32_t L, uint64_t seed,
                             uint32_t epoch, uint32_t batch, int32_t* lid_scratch,
                             uint32_t* uniq, uint64_t uniq_cap, uint64_t* sizes,
                             uint32_t* blk_indptr, uint64_t indptr_cap,
                             uint32_t* blk_indices, uint64_t indices_cap, uint64_t* nnz);

/* PinSAGE random-walk neighbour selection ("random
 * walks to select 5 neighbors from 4 paths of length 3"; reading Q13) +
 * the same relabel.  blk_weights parallels blk_indices (visit counts). */
int orc_sample_rwalk(const uint64_t* indptr, const uint32_t* indices, uint64_t V,
                     const uint32_t* seeds, uint64_t n0, uint32_t L, uint32_t walks,
                     uint32_t walk_len, uint32_t topk, uint64_t seed, uint32_t epoch,
                     uint32_t batch, int32_t* lid_scratch, uint32_t* uniq, uint64_t uniq_cap,
                     uint64_t* sizes, uint32_t* blk_indptr, uint64_t indptr_cap,
                     uint32_t* blk_indices, uint32_t* blk_weights, uint64_t indices_cap,
                     uint64_t* nnz);

/* Random policy hotness (L442): hi32(draw64(v,0,0,c3(0,0,7),0)) for every vertex. */
void orc_policy_random(uint64_t seed, uint64_t V, uint32_t* out);

/* Extract (Fig 9): out[i,:] = features[vertices[i],:]. */
int orc_extract(const float* features, uint64_t V, uint32_t D, const uint32_t* vertices,
                uint64_t n, float* out);

#ifdef __cplusplus
}
#endif
#endif
