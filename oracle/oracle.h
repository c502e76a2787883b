/* oracle.h — plain, slow, single-threaded CPU oracle for the HEC hot path.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load this library.  It shares no
 * code, header, table or helper with the CUDA path (paper_conf_ipps_gilbertabmr21_b200/).
 *
 * What it computes (PAPER.md = /root/reference/PAPER.md):
 *   oracle_heavy      : Alg 3 lines 6-10 / Alg 4 lines 3-8 (PAPER.md:L109-119,
 *                       L177-187): H[u] = first neighbour of maximum weight with
 *                       a strict ">" scan from w = 0 (sorted columns => smallest id).
 *   oracle_prio       : the visit order P of GENPERM, fixed by R3
 *                       (splitmix64 priorities; reading Z2).
 *   oracle_mapping    : Alg 3 verbatim, visit in ascending
 *                       priority, then coarse ids renumbered by ascending root id
 *                       (FINDUNIQANDRELABEL; reading Z3).
 *   oracle_coarsen    : the plain definition A_c = P A P^T with
 *                       the diagonal dropped ("We omit counting self-loops",
 *                       PAPER.md:L280); rows list ascending coarse columns.
 * All ids are 0-based; row offsets int64, ids/weights int32 (R7).
 */
#ifndef HEC_ORACLE_H
#define HEC_ORACLE_H
#include <stdint.h>

#define ORACLE_OK 0
#define ORACLE_EINVAL (-1)
#define ORACLE_ENOMEM (-2)
#define ORACLE_EOVERFLOW (-4)

uint64_t oracle_splitmix64(uint64_t x);
/* prio_l(u) = (splitmix64(s_l ^ u) >> 32) << 32 | u,  s_l = splitmix64(seed + level) */
uint64_t oracle_prio(uint64_t seed, int level, int64_t u);
void oracle_prio_fill(uint64_t seed, int level, int64_t n, uint64_t *prio);

void oracle_heavy(int64_t n, const int64_t *row_ptr, const int32_t *col,
                  const int32_t *wgt, int32_t *H);

/* prio: n distinct priorities (the visit order is ascending prio).
 * M (out, n), *n_c (out).  root (out, optional, n bytes): 1 for aggregate roots. */
int oracle_mapping(int64_t n, const int64_t *row_ptr, const int32_t *col,
                   const int32_t *wgt, const uint64_t *prio, int32_t *M,
                   int64_t *n_c, uint8_t *root);

/* HEC3 (Alg 5): the order-free second phase of HEC.
 * Mutual heavy neighbours collapse onto the smaller id (l.5-8), every heavy
 * neighbour not yet mapped becomes its own root (l.9-12), the remaining
 * vertices inherit their heavy neighbour's (l.13-16), pointer jumping to the
 * root (l.17-21), FINDUNIQANDRELABEL by ascending root id (l.22, reading Z3).
 * P is the identity (reading Z17: Alg 5's O only renames vertices).
 * M (out, n), *n_c (out), root (out, optional, n bytes). */
int oracle_mapping_hec3(int64_t n, const int64_t *row_ptr, const int32_t *col,
                        const int32_t *wgt, int32_t *M, int64_t *n_c, uint8_t *root);

/* HEM (Alg 2) verbatim: vertices visited in ascending prio;
 * an unmatched u takes its heaviest unmatched neighbour (strict ">" from 0:
 * the smallest id among equal maxima) or stays a singleton.  Coarse ids by
 * ascending root id, the root being the visiting vertex u (reading Z3). */
int oracle_mapping_hem(int64_t n, const int64_t *row_ptr, const int32_t *col,
                       const int32_t *wgt, const uint64_t *prio, int32_t *M,
                       int64_t *n_c, uint8_t *root);

/* Output arrays are caller-allocated with the upper bounds row_ptr_c[n_c+1],
 * col_c[nnz], wgt_c[nnz], vwgt_c[n_c]; *nnz_c receives the coarse entry count.
 * *intra receives the directed weight of dropped self-loops (conservation). */
int oracle_coarsen(int64_t n, const int64_t *row_ptr, const int32_t *col,
                   const int32_t *wgt, const int32_t *vwgt, const int32_t *M,
                   int64_t n_c, int64_t *row_ptr_c, int32_t *col_c,
                   int32_t *wgt_c, int32_t *vwgt_c, int64_t *nnz_c,
                   int64_t *intra);
#endif
