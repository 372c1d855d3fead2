/*
 * epi4.h — C ABI of libepi4, the B200 (sm_100a) exhaustive fourth-order K2 epistasis search.
 *
 * The boundary of the hot path.  Plain C types only: no torch types, host or
 * device pointers plus sizes.  Every step of the search runs in libepi4's CUDA kernels; the thin
 * Python binding (paper_conf_icpp_nobreiss22_b200/binding.py) only marshals arguments.
 *
 * Notation (repo naming; PAPER.md swaps the symbols):
 *   N  = number of SNPs (PAPER.md's M), 4 <= N <= 65536 (16-bit SNP indices)
 *   n0 = controls, n1 = cases, M = n0 + n1 samples (PAPER.md's N0, N1, N).
 *
 * Errors: every int-returning call returns 0 on success or a negative EPI4_E* code; the message
 * of the last failure on the calling thread is available from epi4_last_error().  No call
 * throws, aborts or exits across the ABI.
 *
 * Threading: a context is used by one host thread at a time.  One context per GPU / rank.
 */
#ifndef EPI4_H
#define EPI4_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* ---- error codes ---------------------------------------------------------------------- */
#define EPI4_OK       0
#define EPI4_EINVAL  (-1)  /* bad argument: N<4 or N>65536, n_controls<1 or n_cases<1, top_k out of
                              range, pad bits set, AA&Aa != 0, genotype code > 2, phenotype > 1 */
#define EPI4_ENOMEM  (-2)  /* device or host allocation failed (incl. tables too large for HBM) */
#define EPI4_ECUDA   (-3)  /* a CUDA runtime call or kernel failed */
#define EPI4_ESTATE  (-4)  /* call out of order, e.g. search before any load */
#define EPI4_ENODEV  (-5)  /* no sm_100 device / the requested device is unusable */

/* ---- options ---------------------------------------------------------------------------- */
#define EPI4_PIPE_TC    0  /* tcgen05.mma.cta_group::2.kind::mxf4 on E2M1 {0,1} nibble tiles, fp32 TMEM accumulators */
#define EPI4_PIPE_LOP3  1  /* CUDA-core LOP3 (AND) + POPC contraction (cross-check path) */

#define EPI4_PTR_HOST   0
#define EPI4_PTR_DEVICE 1

#define EPI4_MAX_TOPK   1024

typedef struct epi4_ctx epi4_ctx;   /* opaque; owns its device memory and CUDA stream */

typedef struct {
    int32_t block;    /* SNP block size B.  Only 32 is supported.            */
    int32_t pipe;     /* EPI4_PIPE_*                                                               */
    int32_t rank;     /* this process' rank and the world size: epi4_search evaluates only the     */
    int32_t world;    /*   work units the static LPT plan assigns to `rank`       */
    int32_t grid;     /* persistent-kernel CTAs (0 = number of SMs, rounded down to whole CTA pairs)  */
    int32_t debug;    /* 0 in production.  Bit 16 = exact score for every quad (no fp32 filter; exact */
                      /*   results).  Other bits disable warp roles (results invalid) and are only    */
                      /*   accepted by a diagnostics build (EPI4_DEBUG_MODES), else EPI4_EINVAL.      */
    int32_t flags;    /* EPI4_FLAG_* bits                                                          */
    int32_t objective; /* EPI4_OBJ_K2 (default), EPI4_OBJ_MI or EPI4_OBJ_CHI2 (§8(f) NEXT-4) */
} epi4_opts;

/* opts.flags: with world > 1, a load computes only this rank's contiguous share of the 3-way table T3
 * (the triples [rank*S, (rank+1)*S) of the colex order, S = ceil(C(N,3) / world)); the caller all-gathers
 * the shares (epi4_t3_shard / epi4_t3_ready) — the exchange that replaces building T3 on every GPU. */
#define EPI4_FLAG_SHARD_T3 1
/* opts.flags: windowed 3-way table (tensor-core pipe): instead of all C(N,3) triples (32 B each) only two
 * slabs of 128 x C(N,2) triples are resident, rebuilt on the tensor cores during the search;
 * chosen automatically when the resident table does not fit in HBM (e.g. N = 4096), forced by this flag.
 * epi4_tables is unavailable (EPI4_ESTATE) with a windowed table. */
#define EPI4_FLAG_T3_WINDOWED 2
/* opts.flags: tensor-core tile geometry.  By default a load picks N = 224 columns per tile
 * (28 y SNPs; the A operand amortised over more columns, two TMEM accumulator regions) when the dataset has
 * >= 16384 controls or needs 64-bit packed counts, else N = 128 (16 y, three regions, the scoring overlaps
 * both phenotype phases); these flags force one (results are identical, only the speed differs). */
#define EPI4_FLAG_TILE_N128 4
#define EPI4_FLAG_TILE_N224 8

/* opts.objective (the table construction does not depend on the score):
 *   EPI4_OBJ_K2: K2 (the paper's), smallest first.
 *   EPI4_OBJ_MI: mutual information between the quad's 81-cell genotype and the phenotype, largest first.
 *     Computed exactly as M*I = sum_c [(X(r_c0) + X(r_c1)) - X(r_c)] + (X(M) - X(n0) - X(n1)) with
 *     X(k) = k ln k (X(0) = 0) from a host-built double table, summed in canonical cell order; the key
 *     returned in k2_out is -M*I (so "smallest key first" ranks by largest MI).  The tensor-core pipe skips
 *     quads whose fp32 upper bound on M*I cannot reach the top-k (rigorous rounding bound; exact result).
 *     epi4_search3 ranks triples by the same objective (27 cells, exact, no filter). */
#define EPI4_OBJ_K2 0
#define EPI4_OBJ_MI 1
/*   EPI4_OBJ_CHI2: Pearson's chi-square of the 2 x 81 table (no continuity correction, cells with r_c > 0),
 *     largest first, computed as X^2 = M*S/(n0 n1) - M with S = sum_{c: r_c>0} (r_c0^2 n1 + r_c1^2 n0) / r_c:
 *     an exact integer numerator (uint64, < n0 n1 M), one correctly rounded double division per cell, summed in
 *     canonical cell order; X^2 = 0 if a phenotype is empty.  The key in k2_out is -X^2.  epi4_load_* returns
 *     EPI4_EINVAL if n0 n1 M >= 2^53 (the numerator would not be exact in double).  The tensor-core
 *     pipe skips quads whose fp32 upper bound on X^2 cannot reach the top-k (exact result). */
#define EPI4_OBJ_CHI2 2

/* Fill *opts with defaults (block 32, pipe TC, rank 0, world 1, grid 0). */
void epi4_default_opts(epi4_opts* opts);

/* Create a context on CUDA device `cuda_device` (selects it on the calling thread).
 * opts may be NULL (defaults).  *out receives the context; destroy it with epi4_destroy. */
int epi4_create(epi4_ctx** out, int32_t cuda_device, const epi4_opts* opts);
void epi4_destroy(epi4_ctx* ctx);

/* Use `cuda_stream` (a cudaStream_t, e.g. torch.cuda.current_stream().cuda_stream) for all later
 * work of this context; NULL restores the context's own stream. */
int epi4_set_stream(epi4_ctx* ctx, void* cuda_stream);

/* ---- data loading (step a1 of SURVEY.md §8(a); §3.1) --------------------------
 * Bit-packed genotype planes, one matrix per phenotype: row r = 2*snp + g with
 * g = 0 -> AA (homozygous major), g = 1 -> Aa (heterozygous); aa is not stored (inferred).
 * Each row holds ceil(n/32) uint32 words, sample s of that phenotype at bit s%32 of word s/32
 * (LSB first).  Pad bits beyond n must be 0 and AA & Aa must be 0 (checked -> EPI4_EINVAL).
 * The data is copied (the caller keeps ownership).  ptr_kind selects host or device pointers. */
int epi4_load_bits(epi4_ctx* ctx, const uint32_t* planes_ctrl, const uint32_t* planes_case,
                   int32_t n_snps, int64_t n_controls, int64_t n_cases, int32_t ptr_kind);

/* Same, from byte genotypes: geno is N x M, SNP-major, codes {0 = AA, 1 = Aa, 2 = aa};
 * phen[M] is 0 (control) or 1 (case).  The split by phenotype and the bit packing run on the GPU
 * (the pack kernel).  Codes > 2 or phenotypes > 1 -> EPI4_EINVAL. */
int epi4_pack_genotypes(epi4_ctx* ctx, const uint8_t* geno, const uint8_t* phen,
                        int32_t n_snps, int64_t n_samples, int32_t ptr_kind);

/* Copy the packed planes back (host pointers, sized 2*N*ceil(n_p/32) words each). */
int epi4_get_bits(epi4_ctx* ctx, uint32_t* planes_ctrl, uint32_t* planes_case);

/* ---- search (steps a2-a7; Algorithm 1, L109 output s) ------------------------
 * Exhaustive search over every quad i<j<k<l assigned to this rank.  Writes the `top_k` smallest
 * (K2, quad) keys in ascending order (ties -> smaller packed index), K2 in double
 * (readings #1-#4).  Packed quad index:
 * i<<48 | j<<32 | k<<16 | l.  quads_out / k2_out are HOST arrays of top_k entries; *n_out gets
 * min(top_k, number of quads evaluated).  1 <= top_k <= EPI4_MAX_TOPK. */
int epi4_search(epi4_ctx* ctx, int32_t top_k, uint64_t* quads_out, double* k2_out, int32_t* n_out);

/* Search restricted to the work units [unit_begin, unit_end) of this rank's plan (tests, bounded
 * samples of a full-size workload).  unit_end = -1 means "to the end". */
int epi4_search_units(epi4_ctx* ctx, int64_t unit_begin, int64_t unit_end, int32_t top_k,
                      uint64_t* quads_out, double* k2_out, int32_t* n_out);

/* Third-order search (the paper's predecessors): every triple
 * i < j < k of this rank's share (the 4-way plan's units, rank/world as for epi4_search), its 2 x 27 table
 * (8 non-aa counts on the tensor cores against an all-ones SNP, the other 19 recovered from T2/T1/n as in
 * PAPER.md:L126) scored by K2 (or opts.objective) over 27 cells in double, canonical order c = 9a + 3b + c.  Output as
 * epi4_search: the top_k smallest (K2, index) keys ascending, index = i<<48 | j<<32 | k<<16.
 * Tensor-core pipe only (EPI4_EINVAL otherwise); host arrays of top_k entries. */
int epi4_search3(epi4_ctx* ctx, int32_t top_k, uint64_t* triples_out, double* k2_out, int32_t* n_out);

/* Verification hook: the 2 x 81 contingency table (controls row first, cell 27a+9b+3c+d,
 * 0=AA 1=Aa 2=aa) of each listed quad (packed, any SNP order), computed from the device planes:
 * 16 cells by AND+POPC of the planes and the other 65 by the same lower-order recovery the search
 * epilogue uses.  quads and counts_out are host arrays; counts_out has
 * n * 162 entries. */
int epi4_tables(epi4_ctx* ctx, const uint64_t* quads, int64_t n, uint32_t* counts_out);

/* Sharded T3 (opts.flags & EPI4_FLAG_SHARD_T3, world > 1, PAPER.md:L155 builds the tables on
 * every GPU instead).  After a load, *t3_dev receives the device address of the packed T3 buffer (the
 * context owns it), *shard_bytes the size of one rank's share and *total_bytes = world * shard_bytes; this
 * rank's share is already computed at offset rank * shard_bytes.  The caller fills the other shares (an
 * all-gather of equal-size chunks, e.g. NCCL over NVLink) on any stream, synchronizes, and calls
 * epi4_t3_ready.  Until then epi4_search / epi4_tables fail with EPI4_ESTATE.  Without the flag the tables
 * are complete after the load and both calls return EPI4_ESTATE. */
int epi4_t3_shard(epi4_ctx* ctx, void** t3_dev, int64_t* shard_bytes, int64_t* total_bytes);
int epi4_t3_ready(epi4_ctx* ctx);

/* Debug/verification: make the next search also write the 162 counts of EVERY evaluated quad into
 * a device buffer indexed by the quad's colex rank C(l,4)+C(k,3)+C(j,2)+i (162 uint32 each);
 * counts_dev = NULL disables.  Only for small N (the buffer has C(N,4)*162 entries). */
int epi4_set_dump(epi4_ctx* ctx, uint32_t* counts_dev);

/* Verification sample (parity at full size, SURVEY.md §8(c) tier 2): during every later epi4_search /
 * epi4_search_units, record each evaluated quad whose packed index q satisfies
 *     (mix64(q ^ seed) & (2^log2_rate - 1)) == 0,
 *     mix64(x): x ^= x >> 30; x *= 0xBF58476D1CE4E5B9; x ^= x >> 27; x *= 0x94D049BB133111EB; x ^= x >> 31
 * (splitmix64's finalizer, uint64 arithmetic), with its exact key (as in k2_out) and its 2 x 81 table, all
 * computed from the contraction counts of the search kernel itself (the production path, not epi4_tables).
 * Up to `capacity` quads are stored per search (later hits are counted only); capacity = 0 disables.
 * log2_rate = 0 samples every quad.  Device memory is owned by the context. */
int epi4_set_sample(epi4_ctx* ctx, int32_t log2_rate, uint64_t seed, int64_t capacity);
/* Copy the last search's sample to HOST arrays of `capacity` entries (quads, keys; counts: capacity x 162,
 * controls row first as in epi4_tables).  *n_out = number of sampled quads in that search (entries beyond the
 * context's or this call's capacity are not written).  EPI4_ESTATE if no sample is configured.  The order of
 * the entries is unspecified. */
int epi4_get_sample(epi4_ctx* ctx, uint64_t* quads_out, double* keys_out, uint32_t* counts_out, int64_t capacity,
                    int64_t* n_out);

/* ---- plan --------------------------------------------------------------------
 * Work unit u = (w-range, x): all quads whose first SNP lies in [128*wr, 128*wr+128) and
 * whose second SNP is x.  The plan lists this rank's units (static LPT by modelled cost, identical
 * on every rank).  Host-only; usable without a GPU. */
int64_t epi4_plan_count(int32_t n_snps, int32_t rank, int32_t world);
int epi4_plan_units(int32_t n_snps, int32_t rank, int32_t world, int32_t* wb_x_out /* 2 x count */,
                    double* cost_out /* count, may be NULL */);
/* The same with opts.flags: with EPI4_FLAG_T3_WINDOWED the plan a windowed-T3 context uses (whole slab groups
 * (128-SNP range of w, 128-SNP range of x) dealt longest first, groups above 1/(4 world) of the work split by x),
 * so that each rank rebuilds only its own groups' slabs. */
int64_t epi4_plan_count_ex(int32_t n_snps, int32_t rank, int32_t world, int32_t flags);
int epi4_plan_units_ex(int32_t n_snps, int32_t rank, int32_t world, int32_t flags, int32_t* wb_x_out,
                       double* cost_out);

/* ---- measurement ---------------------------------------------------------------------------- */
typedef struct {
    double ms_pack;        /* last load: H2D + pack kernel                         */
    double ms_pop;         /* last load: T1 + T2 + T3 kernels                      */
    double ms_quad;        /* last search: 4-way contraction + fused epilogue      */
    double ms_merge;       /* last search: top-k merge + D2H                       */
    int64_t quads;         /* quads evaluated by the last search (useful)          */
    int64_t tiles;         /* tiles executed by the last search                    */
    int64_t launches;      /* kernels launched by the last search                  */
    int64_t launches_load; /* kernels launched by the last load                    */
    double executed_macs;  /* MACs issued by the last search's contraction (incl. padding/masking) */
    double prof[8];        /* diagnostics: [0] exact-K2 evaluations (filter candidates); with opts.debug
                              & 8 (instrumented build, -DEPI4_PROF) also summed SM cycles: [1] epilogue busy,
                              [2] MMA waiting for the A operand, [3] producer busy, [4] producer waiting for a
                              free B stage, [5] MMA waiting for the B operand, [6] TMA waiting for a free A
                              stage, [7] MMA waiting for a free TMEM region */
    int64_t tile_n;        /* last search: columns per tensor-core tile (128 or 224, EPI4_FLAG_TILE_*); 0 = lop3 */
} epi4_stats;

int epi4_get_stats(epi4_ctx* ctx, epi4_stats* out);

/* Message of the last failure on this thread ("" if none). */
const char* epi4_last_error(void);

/* Library build string (arch, pipe list). */
const char* epi4_version(void);

#ifdef __cplusplus
}
#endif
#endif /* EPI4_H */
