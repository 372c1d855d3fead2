// api.cu — host side of libepi4: the C ABI (include/epi4.h), context and device memory, the
// static LPT work plan, search orchestration and measurement.
//
// Flow of one search (Algorithm 1, L80-L104, re-designed B200-first):
//   load:   H2D of the planes or byte genotypes -> pack / retile kernels -> T1, T2, T3 kernels
//           -> host-built lgamma table (double, "each GPU stores a full copy").
//   search: this rank's units (static LPT) -> tile prefix -> ONE persistent contraction kernel with
//           the fused epilogue over all tiles -> merge of the per-CTA top-k lists -> D2H of top_k.
#include <algorithm>
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <string>
#include <vector>

#include "epi4_internal.cuh"
#include <nvtx3/nvToolsExt.h>   // header-only NVTX v3: host-side phase ranges (ncu --nvtx / Nsight timelines)

namespace {
// one NVTX range per phase of a call: load (pack / retile, tables), search (plan, slab rebuilds, contraction,
// merge), third-order search
struct NvtxRange {
    explicit NvtxRange(const char* name) { nvtxRangePushA(name); }
    ~NvtxRange() { nvtxRangePop(); }
    NvtxRange(const NvtxRange&) = delete;
    NvtxRange& operator=(const NvtxRange&) = delete;
};
}  // namespace

using namespace epi4;

namespace {
thread_local std::string g_err;

int fail(int code, const char* fmt, ...) {
    char buf[512];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof buf, fmt, ap);
    va_end(ap);
    g_err = buf;
    return code;
}

#define CU(call)                                                                                   \
    do {                                                                                           \
        cudaError_t e_ = (call);                                                                   \
        if (e_ != cudaSuccess)                                                                     \
            return fail(e_ == cudaErrorMemoryAllocation ? EPI4_ENOMEM : EPI4_ECUDA, "%s: %s (%s:%d)", \
                        #call, cudaGetErrorString(e_), __FILE__, __LINE__);                        \
    } while (0)

template <class T>
void dfree(T*& p) {
    if (p) cudaFree((void*)p);
    p = nullptr;
}

// grow-only device buffer: reallocates only when a larger size is needed (loads of same-shaped
// datasets reuse every allocation, so a step does no cudaMalloc/cudaFree)
template <class T>
cudaError_t grow(T*& p, size_t& cap, size_t bytes) {
    if (bytes <= cap && p) return cudaSuccess;
    if (p) cudaFree((void*)p);
    p = nullptr;
    cap = 0;
    cudaError_t e = cudaMalloc((void**)&p, bytes ? bytes : 16);
    if (e == cudaSuccess) cap = bytes;
    return e;
}
}  // namespace

// The work plan of a search, cached across searches of the same shape: a bench step re-plans nothing and copies
// no plan data to the device.  This rank's units [ub, ue) of the static LPT plan, grouped by slab (R, X) when the
// 3-way table is windowed, with their group-relative inclusive prefix of tiles; the tile table of a one-group,
// one-chunk plan stays on the device.
struct SearchPlan {
    struct Group { int64_t b, e; int32_t wr, xr; };
    bool valid = false;
    int32_t n = 0, rank = 0, world = 0, pipe = -1;
    int64_t ub = 0, ue = 0;
    bool windowed = false;
    int32_t yr = 0;                     // y-range of the tiles the prefix counts
    std::vector<Unit> units;
    std::vector<int64_t> prefix;        // group-relative inclusive prefix of tiles per unit
    std::vector<Group> groups;
    bool table_cached = false;
};

struct epi4_ctx {
    int device = 0;
    epi4_opts opts{};
    int sm_count = 0;
    cudaStream_t own_stream = nullptr, stream = nullptr;
    // dataset
    bool loaded = false;
    bool t3_pending = false;       // sharded T3: the other ranks' shares are not in yet (epi4_t3_ready)
    int64_t t3_shard = 0;          // triples per rank share (sharded) or C(N,3)
    int32_t n = 0, npad = 0;
    int64_t np[2] = {0, 0};
    int32_t nchunks[2] = {0, 0};
    int32_t tc_yr = EPI4_YR_N128;  // tensor-core tile geometry of this dataset (y per tile: N = 8 tc_yr; tc_tile_yr)
    uint32_t* planes[2] = {nullptr, nullptr};
    uint32_t *T1 = nullptr, *T2 = nullptr, *T3 = nullptr;
    uint32_t* T3x = nullptr;       // windowed T3: the slab FIRST(X) (T3 then holds FIRST(R))
    size_t cap_T3x = 0;
    bool t3_windowed = false;
    double* lgam = nullptr;
    double* xlx = nullptr;         // X(k) = k ln k (EPI4_OBJ_MI)
    size_t cap_xlx = 0;
    std::vector<double> host_X;
    uint8_t* expl[2] = {nullptr, nullptr};
    size_t cap_planes[2] = {0, 0}, cap_T1 = 0, cap_T2 = 0, cap_T3 = 0, cap_lgam = 0, cap_expl[2] = {0, 0};
    unsigned char* scratch = nullptr;     // H2D staging / pack indices
    std::vector<double> host_L;           // lgamma(n + 1), grown on demand
    std::vector<uint64_t> host_tiles;     // 3-way-table mode / third-order search tile lists
    uint64_t* d_tiles3 = nullptr;         // device copy of a host-built tile list
    size_t cap_tiles3 = 0;
    int64_t t3_tiles_key = -1;            // d_tiles3 holds the resident-T3 tiles of this N (no rebuild per load)
    int64_t t3_tiles_n = 0;
    int64_t lgam_m = -1, xlx_m = -1;      // M of the tables currently on the device (uploaded once per M)
    size_t cap_scratch = 0;
    // search workspace
    Unit* d_units = nullptr;
    int64_t* d_prefix = nullptr;
    size_t units_cap = 0;
    SearchPlan plan;
    int64_t tile_chunk = (int64_t)1 << 25;   // tiles per search launch (bounds the tile table: 256 MiB)
    uint64_t* d_tiles = nullptr;   // tensor-core pipe: decoded tile table (k_tile_table), 8 B per tile
    size_t cap_tiles = 0;
    unsigned long long* d_counters = nullptr;   // [0] tile counter, [1] quads done
    double* d_list_k2 = nullptr;
    uint64_t* d_list_idx = nullptr;
    int32_t* d_list_cnt = nullptr;
    size_t list_entries = 0;
    int32_t list_slots = 0;
    double* d_out_k2 = nullptr;
    uint64_t* d_out_idx = nullptr;
    int32_t* d_out_n = nullptr;
    unsigned int* d_status = nullptr;
    uint32_t* dump = nullptr;
    unsigned char* h_out = nullptr;       // pinned: small device -> host results (counts, status, counters)
    // verification sample (epi4_set_sample)
    int64_t samp_cap = 0;
    uint64_t samp_seed = 0, samp_mask = 0;
    unsigned long long* d_samp_n = nullptr;
    uint64_t* d_samp_idx = nullptr;
    double* d_samp_key = nullptr;
    uint32_t* d_samp_counts = nullptr;
    cudaEvent_t ev[6] = {};
    epi4_stats stats{};
};

namespace {

// Offset of the fp32 K2 filter (epilogue.cuh, reading #16): a quad is scored exactly iff
// ln2 A + off <= threshold, off = -81 - 81 C0 - 13.5 - E(M): K2 - (ln2 A_exact - 81 - 81 C0) > -13.5 (Stirling
// remainder) and E(M) bounds ln2 |A - A_exact| from fp32 arithmetic (A in log2 units).  Over a quad's 243
// terms, sum (k + 1/2) <= 2M + 203 and every argument is <= M + 2:
//   lg2.approx: absolute error <= 2^-21 max(1, log2(M + 2)), times the coefficient (k + 1/2);
//   accumulation: every cell adds its three terms to one of three running sums by FFMA (or, with
//   EPI4_FILTER_F2, one of the two lanes of an FFMA2 pair, epilogue.cuh cell_T_acc2; 243 roundings either way); a
//   running sum is at most P = M + 81 (log2(M + 2) + 2) between cells and at most P + (n + 3/2) log2(M + 2)
//   inside a cell, so the roundings total <= u (243 P + 3 (M + 122) log2(M + 2)); + 2 final adds of <= P.
// E is doubled for safety; at M = 16384 E ~ 0.6, at M = 100003 ~ 4.
double filter_offset(int64_t m) {
    const double M = (double)m, u = std::ldexp(1.0, -24), l2M = std::log2(M + 2.0), ln2 = std::log(2.0);
    const double e_log = std::ldexp(1.0, -21) * std::max(1.0, l2M) * (2.0 * M + 203.0);
    const double P = M + 81.0 * (l2M + 2.0);
    const double e_cell = 3.0 * u * (M + 122.0) * l2M;
    const double e_acc = (243.0 + 2.0) * u * P;
    const double E = 2.0 * ln2 * (e_log + e_cell + e_acc);
    const double C0 = 0.5 * std::log(2.0 * M_PI) - 1.0;
    return -81.0 - 81.0 * C0 - 13.5 - E;
}

// 32-bit packed words need c0 < 2^bits(n0) and bits(n0) + bits(n1) <= 32 (and counts < 2^22 for the fp32
// exponent trick); beyond that every table and epilogue word is 64-bit (c0 | c1 << 32)
int bits_of(int64_t v) { int b = 1; while (b < 62 && ((int64_t)1 << b) <= v) ++b; return b; }
bool is_wide(int64_t n0, int64_t n1) {
    return bits_of(n0) + bits_of(n1) > 32 || n0 >= ((int64_t)1 << 22) || n1 >= ((int64_t)1 << 22);
}

DevData devdata(const epi4_ctx* c) {
    DevData d;
    d.planes[0] = c->planes[0];
    d.planes[1] = c->planes[1];
    d.nchunks[0] = c->nchunks[0];
    d.nchunks[1] = c->nchunks[1];
    d.nchunks4[0] = (c->nchunks[0] + 1) / 2;
    d.nchunks4[1] = (c->nchunks[1] + 1) / 2;
    d.nrb = c->npad / 64;
    // c0 <= n0 < 2^pk_shift; 16 whenever both counts fit 16 bits (the epilogue then unpacks each half into a
    // float with one byte permute, epilogue.cuh cell_T_acc<true>)
    d.pk_shift = 1;
    while (d.pk_shift < 31 && ((int64_t)1 << d.pk_shift) <= c->np[0]) ++d.pk_shift;
    if (c->np[0] < 65536 && c->np[1] < 65536) d.pk_shift = 16;
    // wide: the two counts do not fit one 32-bit word -> 64-bit packed words (c0 | c1 << 32) everywhere
    d.wide = is_wide(c->np[0], c->np[1]) ? 1 : 0;
    if (d.wide) d.pk_shift = 32;
    d.n = c->n;
    d.npad = c->npad;
    d.np[0] = (uint32_t)c->np[0];
    d.np[1] = (uint32_t)c->np[1];
    d.npk = d.wide ? 0u : (uint32_t)c->np[0] | ((uint32_t)c->np[1] << d.pk_shift);
    d.T1 = c->T1;
    d.T2 = c->T2;
    d.T3 = c->T3;
    d.T3x = c->T3;
    d.t3_win = 0;
    d.t3_w0 = d.t3_x0 = 0;
    d.lgam = c->lgam;
    d.xlx = c->xlx;
    d.objective = c->opts.objective;
    {
        const double M = (double)(c->np[0] + c->np[1]), a = (double)c->np[0], b = (double)c->np[1];
        d.mi_const = (M > 0 ? M * std::log(M) : 0.0) - (a > 0 ? a * std::log(a) : 0.0) - (b > 0 ? b * std::log(b) : 0.0);
    }
    d.expl[0] = c->expl[0];
    d.expl[1] = c->expl[1];
    d.flt_off = filter_offset(c->np[0] + c->np[1]);
    {
        const double M = (double)(c->np[0] + c->np[1]);
        d.chi_a = c->np[0] ? (float)(M / (double)c->np[0]) : 0.0f;
        d.chi_b = c->np[1] ? (float)(M / (double)c->np[1]) : 0.0f;
        d.chi_M = M;
        // MI filter bound (epilogue.cuh cell_mi): lg2.approx calls (coefficients sum to 2M), the three
        // roundings of each cell (each <= u * r_c lg2 r_c, sum <= 3 u M lg2 M), and 29 additions of the cell
        // values (|cell| <= r_c bits, so the partial sums are <= M); doubled, as for the K2 filter
        const double u = std::ldexp(1.0, -24), l2M = std::log2(M + 2.0);
        d.mi_E = 2.0 * (std::ldexp(1.0, -21) * std::max(1.0, l2M) * (2.0 * M + 243.0) + 3.0 * u * (M + 81.0) * l2M +
                        29.0 * u * (M + 81.0));
    }
    return d;
}

void release_data(epi4_ctx* c) {
    dfree(c->scratch);
    dfree(c->planes[0]);
    dfree(c->planes[1]);
    dfree(c->T1);
    dfree(c->T2);
    dfree(c->T3);
    dfree(c->T3x);
    dfree(c->lgam);
    dfree(c->xlx);
    dfree(c->expl[0]);
    dfree(c->expl[1]);
    c->loaded = false;
}

// ---- plan: units, modelled cost, static LPT --------------------------------------------------------
struct PlanEntry {
    Unit u;
    double cost;
};

std::vector<PlanEntry> all_units(int32_t n) {
    std::vector<PlanEntry> v;
    const int32_t nr = (n + EPI4_WP - 1) / EPI4_WP;
    for (int32_t wr = 0; wr < nr; ++wr)
        for (int32_t x = wr * EPI4_WP + 1; x <= n - 3; ++x) {
            const double cost = (double)unit_tiles(n, x);
            if (cost > 0) v.push_back({{wr, x}, cost});
        }
    return v;
}

// Slab group of a unit for the windowed 3-way table: (128-SNP range of w, 128-SNP range of x) — a launch over one
// group reads only the slabs FIRST(R) and FIRST(X).
inline int64_t slab_group(const Unit& u) { return (int64_t)u.wr * 65536 + u.x / EPI4_WP; }

// Static LPT plan of this rank, identical on every rank.  grouped = false: units dealt longest
// first onto the least-loaded rank.  grouped = true (windowed T3): whole slab groups (R, X) are dealt longest
// first, so a rank rebuilds only the slabs of its own groups (~groups / world of them instead of all); a group
// larger than 1/(4 world) of the total is split into x sub-ranges first so that the partition stays balanced.
std::vector<PlanEntry> plan_rank(int32_t n, int32_t rank, int32_t world, bool grouped = false) {
    std::vector<PlanEntry> v = all_units(n);
    // longest processing time first; ties broken by (wb, x) so every rank computes the same plan
    std::stable_sort(v.begin(), v.end(), [](const PlanEntry& a, const PlanEntry& b) {
        if (a.cost != b.cost) return a.cost > b.cost;
        if (a.u.wr != b.u.wr) return a.u.wr < b.u.wr;
        return a.u.x < b.u.x;
    });
    if (world <= 1) return v;
    std::vector<double> load(world, 0.0);
    std::vector<PlanEntry> mine;
    if (!grouped) {
        for (const PlanEntry& e : v) {
            int best = 0;
            for (int r = 1; r < world; ++r)
                if (load[r] < load[best]) best = r;
            load[best] += e.cost;
            if (best == rank) mine.push_back(e);
        }
        return mine;
    }
    // groups of units in (R, X) order, big groups split into consecutive-x pieces of <= cap cost
    std::stable_sort(v.begin(), v.end(), [](const PlanEntry& a, const PlanEntry& b) {
        const int64_t ga = slab_group(a.u), gb = slab_group(b.u);
        if (ga != gb) return ga < gb;
        return a.u.x < b.u.x;
    });
    double total = 0.0;
    for (const PlanEntry& e : v) total += e.cost;
    const double cap = total / (4.0 * world);
    struct Piece { size_t b, e; double cost; };
    std::vector<Piece> pieces;
    for (size_t i = 0; i < v.size(); ++i) {
        const bool same = !pieces.empty() && slab_group(v[pieces.back().b].u) == slab_group(v[i].u);
        if (!same || pieces.back().cost + v[i].cost > cap) pieces.push_back(Piece{i, i, 0.0});
        pieces.back().e = i + 1;
        pieces.back().cost += v[i].cost;
    }
    std::vector<size_t> order(pieces.size());
    for (size_t i = 0; i < order.size(); ++i) order[i] = i;
    std::stable_sort(order.begin(), order.end(), [&](size_t a, size_t b) { return pieces[a].cost > pieces[b].cost; });
    for (size_t k : order) {
        int best = 0;
        for (int r = 1; r < world; ++r)
            if (load[r] < load[best]) best = r;
        load[best] += pieces[k].cost;
        if (best == rank)
            for (size_t i = pieces[k].b; i < pieces[k].e; ++i) mine.push_back(v[i]);
    }
    return mine;
}

int ensure_lists(epi4_ctx* c, int32_t slots, int32_t cap) {
    const size_t need = (size_t)slots * cap;
    if (need > c->list_entries) {
        dfree(c->d_list_k2);
        dfree(c->d_list_idx);
        CU(cudaMalloc(&c->d_list_k2, need * sizeof(double)));
        CU(cudaMalloc(&c->d_list_idx, need * sizeof(uint64_t)));
        c->list_entries = need;
    }
    if (slots > c->list_slots) {
        dfree(c->d_list_cnt);
        CU(cudaMalloc(&c->d_list_cnt, (size_t)slots * sizeof(int32_t)));
        c->list_slots = slots;
    }
    return 0;
}

int prepare_units(epi4_ctx* c, int64_t ub, int64_t ue, int32_t G, int32_t YR) {
    SearchPlan& pl = c->plan;
    if (pl.valid && pl.n == c->n && pl.rank == c->opts.rank && pl.world == c->opts.world && pl.pipe == c->opts.pipe &&
        pl.windowed == c->t3_windowed && pl.ub == ub && pl.ue == ue && pl.yr == YR)
        return 0;
    pl.valid = false;
    pl.table_cached = false;
    std::vector<PlanEntry> plan = plan_rank(c->n, c->opts.rank, c->opts.world, c->t3_windowed);
    const int64_t nall = (int64_t)plan.size();
    int64_t b = ub < 0 ? 0 : ub, e = (ue < 0 || ue > nall) ? nall : ue;
    if (b > e) b = e;
    const int64_t nu = e - b;
    pl.units.assign((size_t)nu, Unit{0, 0});
    for (int64_t i = 0; i < nu; ++i) pl.units[(size_t)i] = plan[(size_t)(b + i)].u;
    // Windowed T3: the units are taken grouped by slab (R, X) so that each launch reads only the slabs FIRST(R)
    // and FIRST(X) (rebuilt on the tensor cores when R or X changes); the result does not depend on the order
    // (top-k by (K2, index)).  Resident T3: one group, the plan order.
    pl.groups.clear();
    if (c->t3_windowed && nu > 0) {
        std::stable_sort(pl.units.begin(), pl.units.end(), [](const Unit& p, const Unit& q) {
            const int64_t gp = slab_group(p), gq = slab_group(q);
            return gp != gq ? gp < gq : p.x < q.x;
        });
        for (int64_t i = 0; i < nu; ++i) {
            const Unit& u = pl.units[(size_t)i];
            if (pl.groups.empty() || pl.groups.back().wr != u.wr || pl.groups.back().xr != u.x / EPI4_WP)
                pl.groups.push_back(SearchPlan::Group{i, i, u.wr, u.x / EPI4_WP});
            pl.groups.back().e = i + 1;
        }
    } else if (nu > 0) {
        pl.groups.push_back(SearchPlan::Group{0, nu, -1, -1});
    }
    pl.prefix.assign((size_t)nu, 0);
    int64_t maxg = 0;
    for (const SearchPlan::Group& g : pl.groups) {
        int64_t acc = 0;
        for (int64_t i = g.b; i < g.e; ++i) {
            acc += unit_tiles(c->n, pl.units[(size_t)i].x, YR) * G;
            pl.prefix[(size_t)i] = acc;
        }
        maxg = std::max(maxg, acc);
    }
    if ((size_t)std::max<int64_t>(nu, 1) > c->units_cap) {
        dfree(c->d_units);
        dfree(c->d_prefix);
        c->units_cap = (size_t)std::max<int64_t>(nu, 1);
        CU(cudaMalloc(&c->d_units, c->units_cap * sizeof(Unit)));
        CU(cudaMalloc(&c->d_prefix, c->units_cap * sizeof(int64_t)));
    }
    if (nu > 0) {   // pageable sources: complete when cudaMemcpy returns
        // stream-ordered; pageable sources are staged before cudaMemcpyAsync returns (the vectors may change after)
        CU(cudaMemcpyAsync(c->d_units, pl.units.data(), (size_t)nu * sizeof(Unit), cudaMemcpyHostToDevice, c->stream));
        CU(cudaMemcpyAsync(c->d_prefix, pl.prefix.data(), (size_t)nu * sizeof(int64_t), cudaMemcpyHostToDevice,
                           c->stream));
    }
    if (c->opts.pipe != EPI4_PIPE_LOP3)
        CU(grow(c->d_tiles, c->cap_tiles, (size_t)std::max<int64_t>(1, std::min(maxg, c->tile_chunk)) * sizeof(uint64_t)));
    pl.n = c->n;
    pl.rank = c->opts.rank;
    pl.world = c->opts.world;
    pl.pipe = c->opts.pipe;
    pl.windowed = c->t3_windowed;
    pl.ub = ub;
    pl.ue = ue;
    pl.yr = YR;
    pl.valid = true;
    return 0;
}

// bytes of one windowed-T3 slab: 128 first SNPs x C(n, 2) pairs x 8 packed cells
size_t t3_slab_bytes(int64_t n) { return (size_t)EPI4_WP * (size_t)c2(n) * 8 * sizeof(uint32_t); }

// T3 on the tensor cores (k_quad_tc's 3-way-table mode against the all-ones SNP n, the paper's
// tensorOp_3way): tiles (w-range wp, x, y-range y0, z = n) cover every w < x < y < n exactly
// once.  slab_w0 < 0: all w-ranges, resident colex layout; else only the w-range starting at slab_w0, written
// as the slab FIRST([slab_w0, slab_w0 + 128)) (DevData t3_win).
int build_t3_tc(epi4_ctx* c, uint32_t* out, int32_t slab_w0, int64_t* launches) {
    NvtxRange nvtx_range("epi4: T3 on the tensor cores");
    const int32_t n = c->n;
    // the tile list depends only on (N, slab): the resident list is kept on the device across loads of the same N
    const int64_t key = ((int64_t)n * 2 + (slab_w0 >= 0 ? 1 : 0)) * 64 + c->tc_yr;
    if (slab_w0 >= 0 || c->t3_tiles_key != key) {
        std::vector<uint64_t>& tiles = c->host_tiles;
        tiles.clear();
        for (int32_t x = 1; x <= n - 2; ++x)
            for (int32_t wp = 0; wp * EPI4_WP < x; ++wp) {
                if (slab_w0 >= 0 && wp * EPI4_WP != slab_w0) continue;
                for (int32_t y0 = x + 1; y0 <= n - 1; y0 += c->tc_yr)
                    tiles.push_back((uint64_t)(uint16_t)wp | ((uint64_t)(uint16_t)x << 16) |
                                    ((uint64_t)(uint16_t)y0 << 32) | ((uint64_t)(uint16_t)n << 48));
            }
        c->t3_tiles_key = -1;
        c->t3_tiles_n = (int64_t)tiles.size();
        if (tiles.empty()) return 0;
        CU(grow(c->d_tiles3, c->cap_tiles3, tiles.size() * sizeof(uint64_t)));
        // stream-ordered (a previous slab build on the stream may still read d_tiles3); the pageable source is
        // staged before cudaMemcpyAsync returns, so host_tiles may be rebuilt afterwards
        CU(cudaMemcpyAsync(c->d_tiles3, tiles.data(), tiles.size() * sizeof(uint64_t), cudaMemcpyHostToDevice,
                           c->stream));
        if (slab_w0 < 0) c->t3_tiles_key = key;
    }
    if (c->t3_tiles_n == 0) return 0;
    const int32_t grid = std::max(2, (c->opts.grid > 0 ? c->opts.grid : c->sm_count) / 2 * 2);
    if (int r = ensure_lists(c, grid, 1)) return r;
    SearchParams sp{};
    sp.d = devdata(c);
    sp.yr = c->tc_yr;
    sp.tile_info = c->d_tiles3;
    sp.ntiles = c->t3_tiles_n;
    sp.t3_out = out;
    sp.t3_slab_w0 = slab_w0;
    sp.topk = 1;
    sp.list_k2 = c->d_list_k2;
    sp.list_idx = c->d_list_idx;
    sp.list_cnt = c->d_list_cnt;
    sp.status = c->d_status;
    sp.quads_done = c->d_counters + 2;
    sp.prof = c->d_counters + 24;
    CU(launch_quad_tc(sp, grid, c->stream, launches));
    return 0;
}

// The rest of a load, enqueued behind the pack / retile kernels without waiting for them: tables, expansion,
// T1/T2/T3.  The only host synchronisation of a load is the one at its end, which also reads the status word the
// pack / retile kernels set (invalid genotype codes, pad bits, AA & Aa), so a bad dataset is still rejected by
// the load call itself.
int finish_load(epi4_ctx* c) {
    NvtxRange nvtx_range("epi4: load tables T1/T2/T3");
    // lower-order tables: packed (control | case << pk_shift) words, epilogue.cuh
    {
        // counts become fp32 values 2^23 + r in the filters and pack passes: each class below 2^23 samples
        if (c->np[0] >= ((int64_t)1 << 23) || c->np[1] >= ((int64_t)1 << 23))
            return fail(EPI4_EINVAL, "n0=%lld / n1=%lld: each class must have fewer than 2^23 samples",
                        (long long)c->np[0], (long long)c->np[1]);
        // chi-square: per-cell numerator r_c0^2 n1 + r_c1^2 n0 <= n0 n1 M must be exact in double (epi4.h)
        if (c->opts.objective == EPI4_OBJ_CHI2 &&
            (double)c->np[0] * (double)c->np[1] * (double)(c->np[0] + c->np[1]) >= 9007199254740992.0)
            return fail(EPI4_EINVAL, "EPI4_OBJ_CHI2 needs n0 n1 M < 2^53 (n0=%lld, n1=%lld)", (long long)c->np[0],
                        (long long)c->np[1]);
    }
    const int64_t n = c->n;
    const size_t pw = is_wide(c->np[0], c->np[1]) ? 8 : 4;   // bytes per packed word
    CU(grow(c->T1, c->cap_T1, (size_t)n * 2 * pw));
    CU(grow(c->T2, c->cap_T2, (size_t)c2(n) * 4 * pw));
    const bool shard = (c->opts.flags & EPI4_FLAG_SHARD_T3) && c->opts.world > 1;
    c->t3_shard = shard ? (c3(n) + c->opts.world - 1) / c->opts.world : c3(n);
    const size_t t3b = (size_t)c->t3_shard * (shard ? c->opts.world : 1) * 8 * pw;
    size_t freeb = 0, totb = 0;
    if (t3b > c->cap_T3 || (c->opts.flags & EPI4_FLAG_T3_WINDOWED)) CU(cudaMemGetInfo(&freeb, &totb));   // only when growing
    // windowed T3 (tensor-core pipe): when the resident table does not fit, or on request
    c->t3_windowed = c->opts.pipe == EPI4_PIPE_TC && !shard && n >= 3 &&
                     ((c->opts.flags & EPI4_FLAG_T3_WINDOWED) ||
                      (t3b > c->cap_T3 && t3b + ((size_t)1 << 30) > freeb + c->cap_T3 + c->cap_T3x));
    if (c->t3_windowed) {
        const size_t slab = t3_slab_bytes(n) * (pw / 4);
        CU(grow(c->T3, c->cap_T3, slab));
        CU(grow(c->T3x, c->cap_T3x, slab));
    }
    if (!c->t3_windowed && t3b > c->cap_T3 && t3b + ((size_t)1 << 30) > freeb + c->cap_T3 + c->cap_T3x)
        return fail(EPI4_ENOMEM, "3-way tables need %.1f GB but only %.1f GB of HBM are free (N=%d); "
                    "the windowed T3 needs the tensor-core pipe without sharding", t3b / 1e9, freeb / 1e9, c->n);
    if (!c->t3_windowed) {
        if (c->T3x) {                  // a previous windowed load's FIRST(X) slab: not needed with a resident table
            dfree(c->T3x);
            c->cap_T3x = 0;
        }
        CU(grow(c->T3, c->cap_T3, t3b));
    }
    // lgamma table L[k] = lgamma(k + 1) for k in [0, M + 1]
    const int64_t m = c->np[0] + c->np[1];
    std::vector<double>& L = c->host_L;
    const size_t have = L.size();
    if (have < (size_t)m + 2) {
        L.resize((size_t)m + 2);
        for (size_t k = have; k < L.size(); ++k) L[k] = std::lgamma((double)k + 1.0);
    }
    if (c->lgam_m != m) {   // uploaded once per sample count (stream-ordered; the pageable source is staged)
        CU(grow(c->lgam, c->cap_lgam, ((size_t)m + 2) * sizeof(double)));
        CU(cudaMemcpyAsync(c->lgam, L.data(), ((size_t)m + 2) * sizeof(double), cudaMemcpyHostToDevice, c->stream));
        c->lgam_m = m;
    }
    if (c->opts.objective == EPI4_OBJ_MI) {   // X(k) = k ln k, X(0) = 0
        std::vector<double>& X = c->host_X;
        const size_t hx = X.size();
        if (hx < (size_t)m + 2) {
            X.resize((size_t)m + 2);
            for (size_t k = hx; k < X.size(); ++k) X[k] = k ? (double)k * std::log((double)k) : 0.0;
        }
        if (c->xlx_m != m) {
            CU(grow(c->xlx, c->cap_xlx, ((size_t)m + 2) * sizeof(double)));
            CU(cudaMemcpyAsync(c->xlx, X.data(), ((size_t)m + 2) * sizeof(double), cudaMemcpyHostToDevice, c->stream));
            c->xlx_m = m;
        }
    }
    CU(cudaEventRecord(c->ev[2], c->stream));
    // the tensor-core pipe builds T3 on the tensor cores (k_quad_tc's 3-way-table mode, the paper's
    // tensorOp_3way) against the all-ones SNP n; the CUDA-core pipe and the sharded
    // multi-GPU load keep the POPC kernel (k_pop3), an independent path
    const bool t3_tc = c->opts.pipe == EPI4_PIPE_TC && !shard && n >= 3;
    for (int p = 0; p < 2; ++p) {
        if (c->opts.pipe == EPI4_PIPE_TC && n >= 3)   // z of the 3-way-table mode and the third-order search
            CU(launch_ones_plane(c->planes[p], (int32_t)n, c->npad, c->nchunks[p], c->np[p], c->stream,
                                 &c->stats.launches_load));
        CU(grow(c->expl[p], c->cap_expl[p], (size_t)(((c->nchunks[p] + 1) / 2 + 1) / 2 * 2) * c->npad * 2 * 128));   // fp4 rows
        CU(launch_expand(c->planes[p], c->npad, c->nchunks[p], c->expl[p], c->stream, &c->stats.launches_load));
    }
    {
        const int64_t lo = shard ? std::min<int64_t>(c3(n), (int64_t)c->opts.rank * c->t3_shard) : 0;
        const int64_t hi = t3_tc ? 0 : shard ? std::min<int64_t>(c3(n), lo + c->t3_shard) : c3(n);
        CU(launch_pop(devdata(c), c->T1, c->T2, c->T3, t3_tc ? 0 : lo, hi, c->stream, &c->stats.launches_load));
    }
    if (t3_tc && !c->t3_windowed) {
        if (int r = build_t3_tc(c, c->T3, -1, &c->stats.launches_load)) return r;
    }
    CU(cudaEventRecord(c->ev[3], c->stream));
    unsigned int* st_h = reinterpret_cast<unsigned int*>(c->h_out + 8);
    CU(cudaMemcpyAsync(st_h, c->d_status, sizeof(unsigned int), cudaMemcpyDeviceToHost, c->stream));
    CU(cudaStreamSynchronize(c->stream));   // the load's one host synchronisation
    const unsigned int st = *st_h;
    if (st & EPI4_ST_BAD_GENO) return fail(EPI4_EINVAL, "genotype code > 2");
    if (st & EPI4_ST_BAD_PHEN) return fail(EPI4_EINVAL, "phenotype value > 1");
    if (st & EPI4_ST_PAD_BITS) return fail(EPI4_EINVAL, "pad bits beyond the sample count are set");
    if (st & EPI4_ST_AA_AND_Aa) return fail(EPI4_EINVAL, "a sample has both AA and Aa bits set");
    float ms = 0;
    CU(cudaEventElapsedTime(&ms, c->ev[2], c->ev[3]));
    c->stats.ms_pop = ms;
    c->loaded = true;
    c->t3_pending = shard;
    return 0;
}

}  // namespace

extern "C" int epi4_t3_shard(epi4_ctx* c, void** t3_dev, int64_t* shard_bytes, int64_t* total_bytes) {
    if (!c || !t3_dev || !shard_bytes || !total_bytes) return fail(EPI4_EINVAL, "NULL argument");
    if (!c->loaded) return fail(EPI4_ESTATE, "no data loaded");
    if (!((c->opts.flags & EPI4_FLAG_SHARD_T3) && c->opts.world > 1))
        return fail(EPI4_ESTATE, "T3 is not sharded (opts.flags & EPI4_FLAG_SHARD_T3 with world > 1)");
    *t3_dev = c->T3;
    *shard_bytes = c->t3_shard * 8 * (int64_t)(is_wide(c->np[0], c->np[1]) ? 8 : 4);
    *total_bytes = *shard_bytes * c->opts.world;
    return 0;
}

extern "C" int epi4_t3_ready(epi4_ctx* c) {
    if (!c) return fail(EPI4_EINVAL, "ctx is NULL");
    if (!c->loaded || !c->t3_pending) return fail(EPI4_ESTATE, "no sharded T3 pending");
    c->t3_pending = false;
    return 0;
}

namespace {

// Tensor-core tile geometry (k_quad_tc.cuh): N = 224 columns amortise the A operand over 1.75x the
// columns but leave room for only two TMEM regions, so the scoring of a tile overlaps only the first (control)
// phase of the next; N = 128 keeps three regions.  Measured on one B200 (profiles/r02f_variants.log,
// r02g_geom_ab.log, r02s_c3_geom.log): N = 224 is 7 % faster on the full C5 search (70002 controls), 4 % on the
// full C3 search (16384 controls: 150.0 vs 156.2 s) and 17 % slower with 8192 (C2).  The wide (64-bit packed) mode has two regions in
// both geometries.  opts.flags can force either.
int32_t tc_tile_yr(int32_t flags, int64_t n0, int64_t n1) {
    if (flags & EPI4_FLAG_TILE_N224) return EPI4_YR_N224;
    if (flags & EPI4_FLAG_TILE_N128) return EPI4_YR_N128;
    return (n0 >= 16384 || is_wide(n0, n1)) ? EPI4_YR_N224 : EPI4_YR_N128;
}

int alloc_planes(epi4_ctx* c, int32_t n, int64_t n0, int64_t n1) {
    c->loaded = false;
    c->n = n;
    c->npad = (n + EPI4_YR_MAX + EPI4_WP - 1) / EPI4_WP * EPI4_WP;   // rows past n read as zero planes
    c->np[0] = n0;
    c->np[1] = n1;
    c->tc_yr = tc_tile_yr(c->opts.flags, n0, n1);
    for (int p = 0; p < 2; ++p) {
        c->nchunks[p] = (int32_t)((c->np[p] + EPI4_CHUNK_SAMPLES - 1) / EPI4_CHUNK_SAMPLES);
        const size_t words = (size_t)c->nchunks[p] * c->npad * 2 * EPI4_CHUNK_WORDS;
        CU(grow(c->planes[p], c->cap_planes[p], words * sizeof(uint32_t)));
        CU(cudaMemsetAsync(c->planes[p], 0, words * sizeof(uint32_t), c->stream));
    }
    CU(cudaMemsetAsync(c->d_status, 0, sizeof(unsigned int), c->stream));
    return 0;
}

int check_dims(int32_t n_snps, int64_t n0, int64_t n1) {
    if (n_snps < 4 || n_snps > 65536) return fail(EPI4_EINVAL, "n_snps=%d outside [4, 65536]", n_snps);
    if (n0 < 1 || n1 < 1) return fail(EPI4_EINVAL, "need at least one control and one case (n0=%lld n1=%lld)",
                                       (long long)n0, (long long)n1);
    if (n0 + n1 > ((int64_t)1 << 31) - 4) return fail(EPI4_EINVAL, "too many samples");
    return 0;
}

}  // namespace

// =====================================================================================================
extern "C" {

void epi4_default_opts(epi4_opts* o) {
    if (!o) return;
    std::memset(o, 0, sizeof *o);
    o->block = EPI4_B;
    o->pipe = EPI4_PIPE_TC;
    o->rank = 0;
    o->world = 1;
    o->grid = 0;
}

const char* epi4_last_error(void) { return g_err.c_str(); }

const char* epi4_version(void) {
    return "libepi4 sm_100a (pipes: tc=tcgen05.mma.cta_group::2.kind::mxf4, lop3=CUDA-core AND+POPC)";
}

int epi4_create(epi4_ctx** out, int32_t cuda_device, const epi4_opts* opts) {
    if (!out) return fail(EPI4_EINVAL, "out is NULL");
    *out = nullptr;
    epi4_opts o;
    epi4_default_opts(&o);
    if (opts) o = *opts;
    if (o.block != EPI4_B) return fail(EPI4_EINVAL, "block=%d: only B=32 is supported", o.block);
    if (o.objective != EPI4_OBJ_K2 && o.objective != EPI4_OBJ_MI && o.objective != EPI4_OBJ_CHI2)
        return fail(EPI4_EINVAL, "objective=%d: EPI4_OBJ_K2, EPI4_OBJ_MI or EPI4_OBJ_CHI2", o.objective);
    if (o.pipe != EPI4_PIPE_TC && o.pipe != EPI4_PIPE_LOP3) return fail(EPI4_EINVAL, "unknown pipe %d", o.pipe);
    if (o.world < 1 || o.rank < 0 || o.rank >= o.world) return fail(EPI4_EINVAL, "bad rank/world %d/%d", o.rank, o.world);
#ifndef EPI4_DEBUG_MODES
    // diagnostic modes that disable warp roles (results invalid) exist only in a diagnostics build
    // (build.py with EPI4_DEBUG_MODES=1); bit 16 (exact score for every quad, results exact) is always allowed
    if (o.debug & ~16) return fail(EPI4_EINVAL, "debug=%d: only bit 16 is available in a production build", o.debug);
#endif
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0) return fail(EPI4_ENODEV, "no CUDA device");
    if (cuda_device < 0 || cuda_device >= ndev) return fail(EPI4_ENODEV, "device %d out of range", cuda_device);
    CU(cudaSetDevice(cuda_device));
    cudaDeviceProp prop;
    CU(cudaGetDeviceProperties(&prop, cuda_device));
    if (prop.major != 10 || prop.minor != 0)
        return fail(EPI4_ENODEV, "device %d is sm_%d%d; libepi4 is built for sm_100a only", cuda_device, prop.major,
                    prop.minor);
    epi4_ctx* c = new epi4_ctx();
    c->device = cuda_device;
    c->opts = o;
    c->sm_count = prop.multiProcessorCount;
    cudaError_t e = cudaStreamCreateWithFlags(&c->own_stream, cudaStreamNonBlocking);
    if (e == cudaSuccess) e = cudaMalloc(&c->d_status, sizeof(unsigned int));
    if (e == cudaSuccess) e = cudaMalloc(&c->d_counters, 32 * sizeof(unsigned long long));
    if (e == cudaSuccess) e = cudaMalloc(&c->d_out_k2, EPI4_MAX_TOPK * sizeof(double));
    if (e == cudaSuccess) e = cudaMalloc(&c->d_out_idx, EPI4_MAX_TOPK * sizeof(uint64_t));
    if (e == cudaSuccess) e = cudaMalloc(&c->d_out_n, sizeof(int32_t));
    for (int i = 0; i < 6 && e == cudaSuccess; ++i) e = cudaEventCreate(&c->ev[i]);
    if (e == cudaSuccess) e = cudaMallocHost(&c->h_out, 512);
    if (e != cudaSuccess) {
        epi4_destroy(c);
        return fail(EPI4_ECUDA, "create: %s", cudaGetErrorString(e));
    }
    c->stream = c->own_stream;
    *out = c;
    return 0;
}

void epi4_destroy(epi4_ctx* c) {
    if (!c) return;
    cudaSetDevice(c->device);
    if (c->stream) cudaStreamSynchronize(c->stream);
    release_data(c);
    dfree(c->d_units);
    dfree(c->d_prefix);
    dfree(c->d_tiles);
    dfree(c->d_tiles3);
    dfree(c->d_counters);
    dfree(c->d_list_k2);
    dfree(c->d_list_idx);
    dfree(c->d_list_cnt);
    dfree(c->d_out_k2);
    dfree(c->d_out_idx);
    dfree(c->d_out_n);
    dfree(c->d_status);
    if (c->h_out) cudaFreeHost(c->h_out);
    dfree(c->d_samp_n);
    dfree(c->d_samp_idx);
    dfree(c->d_samp_key);
    dfree(c->d_samp_counts);
    for (int i = 0; i < 6; ++i)
        if (c->ev[i]) cudaEventDestroy(c->ev[i]);
    if (c->own_stream) cudaStreamDestroy(c->own_stream);
    delete c;
}

int epi4_set_stream(epi4_ctx* c, void* s) {
    if (!c) return fail(EPI4_EINVAL, "ctx is NULL");
    c->stream = s ? (cudaStream_t)s : c->own_stream;
    return 0;
}

int epi4_load_bits(epi4_ctx* c, const uint32_t* pc, const uint32_t* pk, int32_t n_snps, int64_t n0, int64_t n1,
                   int32_t ptr_kind) {
    NvtxRange nvtx_range("epi4_load_bits");
    if (!c) return fail(EPI4_EINVAL, "ctx is NULL");
    c->loaded = false;                    // a rejected load never leaves the previous dataset searchable
    c->t3_pending = false;
    if (!pc || !pk) return fail(EPI4_EINVAL, "planes pointer is NULL");
    if (int r = check_dims(n_snps, n0, n1)) return r;
    CU(cudaSetDevice(c->device));
    c->stats.launches_load = 0;
    if (int r = alloc_planes(c, n_snps, n0, n1)) return r;
    CU(cudaEventRecord(c->ev[0], c->stream));
    const uint32_t* src[2] = {pc, pk};
    if (ptr_kind != EPI4_PTR_HOST && ptr_kind != EPI4_PTR_DEVICE) return fail(EPI4_EINVAL, "ptr_kind %d", ptr_kind);
    const size_t words0 = (size_t)2 * n_snps * (size_t)((c->np[0] + 31) / 32);
    const size_t words1 = (size_t)2 * n_snps * (size_t)((c->np[1] + 31) / 32);
    if (ptr_kind == EPI4_PTR_HOST) CU(grow(c->scratch, c->cap_scratch, (words0 + words1) * sizeof(uint32_t)));
    for (int p = 0; p < 2; ++p) {
        const size_t words = p ? words1 : words0;
        const uint32_t* rows = src[p];
        if (ptr_kind == EPI4_PTR_HOST) {
            uint32_t* tmp = reinterpret_cast<uint32_t*>(c->scratch) + (p ? words0 : 0);
            CU(cudaMemcpyAsync(tmp, src[p], words * sizeof(uint32_t), cudaMemcpyHostToDevice, c->stream));
            rows = tmp;
        }
        CU(launch_retile(rows, n_snps, c->np[p], c->npad, c->nchunks[p], c->planes[p], c->d_status, c->stream,
                         &c->stats.launches_load));
    }
    CU(cudaEventRecord(c->ev[1], c->stream));
    int r = finish_load(c);
    float ms = 0;
    cudaEventElapsedTime(&ms, c->ev[0], c->ev[1]);
    c->stats.ms_pack = ms;
    return r;
}

int epi4_pack_genotypes(epi4_ctx* c, const uint8_t* geno, const uint8_t* phen, int32_t n_snps, int64_t m,
                        int32_t ptr_kind) {
    NvtxRange nvtx_range("epi4_pack_genotypes");
    if (!c) return fail(EPI4_EINVAL, "ctx is NULL");
    c->loaded = false;                    // a rejected load never leaves the previous dataset searchable
    c->t3_pending = false;
    if (!geno || !phen) return fail(EPI4_EINVAL, "genotype pointer is NULL");
    if (n_snps < 4 || n_snps > 65536) return fail(EPI4_EINVAL, "n_snps=%d outside [4, 65536]", n_snps);
    if (m < 2 || m > ((int64_t)1 << 31) - 4) return fail(EPI4_EINVAL, "n_samples=%lld", (long long)m);
    if (ptr_kind != EPI4_PTR_HOST && ptr_kind != EPI4_PTR_DEVICE) return fail(EPI4_EINVAL, "ptr_kind %d", ptr_kind);
    CU(cudaSetDevice(c->device));
    c->stats.launches_load = 0;
    const uint8_t *dg = geno, *dp = phen;
    // class sizes: counted here for host phenotypes (no device round trip), by the split kernel for device ones
    int32_t cnt[2] = {0, 0};
    if (ptr_kind == EPI4_PTR_HOST) {
        for (int64_t s = 0; s < m; ++s) {
            if (phen[s] > 1) return fail(EPI4_EINVAL, "phenotype value > 1");
            ++cnt[phen[s]];
        }
        if (int r = check_dims(n_snps, cnt[0], cnt[1])) return r;
    }
    // scratch: [pack indices (2m+2) int32][genotypes n*m][phenotypes m] (the last two only for host input)
    const size_t idx_bytes = ((size_t)(2 * m + 2) * sizeof(int32_t) + 255) & ~(size_t)255;
    const size_t gbytes = ptr_kind == EPI4_PTR_HOST ? (((size_t)n_snps * m + 255) & ~(size_t)255) + (size_t)m : 0;
    CU(grow(c->scratch, c->cap_scratch, idx_bytes + gbytes));
    int32_t* idx = reinterpret_cast<int32_t*>(c->scratch);   // [m] (idx0 then idx1) + 2 counts
    CU(cudaEventRecord(c->ev[0], c->stream));
    if (ptr_kind == EPI4_PTR_HOST) {
        uint8_t* tg = c->scratch + idx_bytes;
        uint8_t* tp = tg + (((size_t)n_snps * m + 255) & ~(size_t)255);
        CU(cudaMemcpyAsync(tg, geno, (size_t)n_snps * m, cudaMemcpyHostToDevice, c->stream));
        CU(cudaMemcpyAsync(tp, phen, (size_t)m, cudaMemcpyHostToDevice, c->stream));
        dg = tg;
        dp = tp;
    }
    CU(cudaMemsetAsync(c->d_status, 0, sizeof(unsigned int), c->stream));
    // pass 1: split by phenotype (idx0 at [0, m), idx1 at [m, 2m), counts at [2m, 2m+2))
    CU(launch_split_phen(dp, m, idx, idx + m, idx + 2 * m, c->d_status, c->stream, &c->stats.launches_load));
    if (ptr_kind == EPI4_PTR_DEVICE) {   // the sizes decide allocations and launch shapes: one small round trip
        int32_t* h = reinterpret_cast<int32_t*>(c->h_out);
        CU(cudaMemcpyAsync(h, idx + 2 * m, 2 * sizeof(int32_t), cudaMemcpyDeviceToHost, c->stream));
        CU(cudaMemcpyAsync(h + 2, c->d_status, sizeof(unsigned int), cudaMemcpyDeviceToHost, c->stream));
        CU(cudaStreamSynchronize(c->stream));
        if ((uint32_t)h[2] & EPI4_ST_BAD_PHEN) return fail(EPI4_EINVAL, "phenotype value > 1");
        cnt[0] = h[0];
        cnt[1] = h[1];
        if (int r = check_dims(n_snps, cnt[0], cnt[1])) return r;
    }
    if (int r = alloc_planes(c, n_snps, cnt[0], cnt[1])) return r;
    for (int p = 0; p < 2; ++p) {
        cudaError_t e = launch_pack(dg, n_snps, m, idx + (p ? m : 0), c->np[p], c->npad, c->nchunks[p], c->planes[p],
                                    c->d_status, c->stream, &c->stats.launches_load);
        if (e != cudaSuccess) return fail(EPI4_ECUDA, "pack: %s", cudaGetErrorString(e));
    }
    CU(cudaEventRecord(c->ev[1], c->stream));
    const int r = finish_load(c);   // no synchronisation before it: the pack status is read at its end
    float ms = 0;
    cudaEventElapsedTime(&ms, c->ev[0], c->ev[1]);
    c->stats.ms_pack = ms;
    return r;
}

int epi4_get_bits(epi4_ctx* c, uint32_t* pc, uint32_t* pk) {
    if (!c || !pc || !pk) return fail(EPI4_EINVAL, "NULL argument");
    if (!c->loaded) return fail(EPI4_ESTATE, "no data loaded");
    CU(cudaSetDevice(c->device));
    uint32_t* dst[2] = {pc, pk};
    for (int p = 0; p < 2; ++p) {
        const size_t words = (size_t)2 * c->n * (size_t)((c->np[p] + 31) / 32);
        uint32_t* tmp = nullptr;
        CU(cudaMalloc(&tmp, words * sizeof(uint32_t)));
        cudaError_t e = launch_untile(c->planes[p], c->n, c->np[p], c->npad, c->nchunks[p], tmp, c->stream, nullptr);
        if (e == cudaSuccess) e = cudaMemcpyAsync(dst[p], tmp, words * sizeof(uint32_t), cudaMemcpyDeviceToHost, c->stream);
        if (e == cudaSuccess) e = cudaStreamSynchronize(c->stream);
        cudaFree(tmp);
        CU(e);
    }
    return 0;
}

int epi4_set_dump(epi4_ctx* c, uint32_t* counts_dev) {
    if (!c) return fail(EPI4_EINVAL, "ctx is NULL");
    c->dump = counts_dev;
    return 0;
}

int epi4_set_sample(epi4_ctx* c, int32_t log2_rate, uint64_t seed, int64_t capacity) {
    if (!c) return fail(EPI4_EINVAL, "ctx is NULL");
    if (log2_rate < 0 || log2_rate > 63 || capacity < 0) return fail(EPI4_EINVAL, "bad sample arguments");
    CU(cudaSetDevice(c->device));
    dfree(c->d_samp_idx);
    dfree(c->d_samp_key);
    dfree(c->d_samp_counts);
    c->samp_cap = 0;
    if (capacity == 0) return 0;
    if (!c->d_samp_n) CU(cudaMalloc(&c->d_samp_n, sizeof(unsigned long long)));
    CU(cudaMalloc(&c->d_samp_idx, (size_t)capacity * sizeof(uint64_t)));
    CU(cudaMalloc(&c->d_samp_key, (size_t)capacity * sizeof(double)));
    CU(cudaMalloc(&c->d_samp_counts, (size_t)capacity * 162 * sizeof(uint32_t)));
    CU(cudaMemset(c->d_samp_n, 0, sizeof(unsigned long long)));
    c->samp_cap = capacity;
    c->samp_seed = seed;
    c->samp_mask = log2_rate == 0 ? 0 : (~0ull >> (64 - log2_rate));
    return 0;
}

int epi4_get_sample(epi4_ctx* c, uint64_t* quads_out, double* keys_out, uint32_t* counts_out, int64_t capacity,
                    int64_t* n_out) {
    if (!c || !n_out) return fail(EPI4_EINVAL, "NULL argument");
    if (!c->samp_cap) return fail(EPI4_ESTATE, "no verification sample configured (epi4_set_sample)");
    if (capacity < 0 || (capacity > 0 && (!quads_out || !keys_out || !counts_out)))
        return fail(EPI4_EINVAL, "bad output arguments");
    CU(cudaSetDevice(c->device));
    unsigned long long n = 0;
    CU(cudaMemcpyAsync(&n, c->d_samp_n, sizeof n, cudaMemcpyDeviceToHost, c->stream));
    CU(cudaStreamSynchronize(c->stream));
    const int64_t k = std::min<int64_t>(std::min<int64_t>((int64_t)n, capacity), c->samp_cap);
    if (k > 0) {
        CU(cudaMemcpyAsync(quads_out, c->d_samp_idx, (size_t)k * sizeof(uint64_t), cudaMemcpyDeviceToHost, c->stream));
        CU(cudaMemcpyAsync(keys_out, c->d_samp_key, (size_t)k * sizeof(double), cudaMemcpyDeviceToHost, c->stream));
        CU(cudaMemcpyAsync(counts_out, c->d_samp_counts, (size_t)k * 162 * sizeof(uint32_t), cudaMemcpyDeviceToHost,
                           c->stream));
        CU(cudaStreamSynchronize(c->stream));
    }
    *n_out = (int64_t)n;
    return 0;
}

int64_t epi4_plan_count_ex(int32_t n_snps, int32_t rank, int32_t world, int32_t flags) {
    if (n_snps < 4 || n_snps > 65536 || world < 1 || rank < 0 || rank >= world) {
        fail(EPI4_EINVAL, "bad plan arguments");
        return EPI4_EINVAL;
    }
    return (int64_t)plan_rank(n_snps, rank, world, (flags & EPI4_FLAG_T3_WINDOWED) != 0).size();
}

int epi4_plan_units_ex(int32_t n_snps, int32_t rank, int32_t world, int32_t flags, int32_t* out, double* cost_out) {
    if (n_snps < 4 || n_snps > 65536 || world < 1 || rank < 0 || rank >= world || !out)
        return fail(EPI4_EINVAL, "bad plan arguments");
    std::vector<PlanEntry> v = plan_rank(n_snps, rank, world, (flags & EPI4_FLAG_T3_WINDOWED) != 0);
    for (size_t i = 0; i < v.size(); ++i) {
        out[2 * i] = v[i].u.wr;
        out[2 * i + 1] = v[i].u.x;
        if (cost_out) cost_out[i] = v[i].cost;
    }
    return 0;
}

int64_t epi4_plan_count(int32_t n_snps, int32_t rank, int32_t world) { return epi4_plan_count_ex(n_snps, rank, world, 0); }
int epi4_plan_units(int32_t n_snps, int32_t rank, int32_t world, int32_t* out, double* cost_out) {
    return epi4_plan_units_ex(n_snps, rank, world, 0, out, cost_out);
}

int epi4_search_units(epi4_ctx* c, int64_t ub, int64_t ue, int32_t top_k, uint64_t* quads_out, double* k2_out,
                      int32_t* n_out) {
    NvtxRange nvtx_range("epi4_search");
    if (!c) return fail(EPI4_EINVAL, "ctx is NULL");
    if (!c->loaded) return fail(EPI4_ESTATE, "search before any load");
    if (c->t3_pending) return fail(EPI4_ESTATE, "sharded T3 incomplete: all-gather the shares, then epi4_t3_ready");
    if (top_k < 1 || top_k > EPI4_MAX_TOPK) return fail(EPI4_EINVAL, "top_k=%d outside [1, %d]", top_k, EPI4_MAX_TOPK);
    if (!quads_out || !k2_out || !n_out) return fail(EPI4_EINVAL, "NULL output pointer");
    CU(cudaSetDevice(c->device));
    if (c->opts.pipe != EPI4_PIPE_LOP3 && std::max(c->np[0], c->np[1]) > ((int64_t)1 << 24))
        return fail(EPI4_EINVAL, "tensor-core pipe: fp32 accumulators are exact up to 2^24 samples per phenotype "
                                 "(%lld, %lld); use EPI4_PIPE_LOP3", (long long)c->np[0], (long long)c->np[1]);
    const int32_t G = quad_split(c->opts.pipe), YR = c->opts.pipe == EPI4_PIPE_LOP3 ? EPI4_YR : c->tc_yr;
    if (int r = prepare_units(c, ub, ue, G, YR)) return r;
    const SearchPlan& pl = c->plan;
    int32_t grid = c->opts.grid > 0 ? c->opts.grid : c->sm_count;
    grid = std::max(2, grid / 2 * 2);                 // whole CTA pairs
    if (int r = ensure_lists(c, grid, top_k)) return r;
    CU(cudaMemsetAsync(c->d_list_cnt, 0, (size_t)grid * sizeof(int32_t), c->stream));
    CU(cudaMemsetAsync(c->d_counters, 0, 32 * sizeof(unsigned long long), c->stream));
    CU(cudaMemsetAsync(c->d_status, 0, sizeof(unsigned int), c->stream));

    SearchParams sp{};
    sp.d = devdata(c);
    sp.yr = c->tc_yr;
    sp.t3_slab_w0 = -1;
    sp.tile_counter = c->d_counters;
    sp.topk = top_k;
    sp.list_k2 = c->d_list_k2;
    sp.list_idx = c->d_list_idx;
    sp.list_cnt = c->d_list_cnt;
    sp.dump = c->dump;
    sp.samp_cap = c->samp_cap;
    sp.samp_seed = c->samp_seed;
    sp.samp_mask = c->samp_mask;
    sp.samp_n = c->d_samp_n;
    sp.samp_idx = c->d_samp_idx;
    sp.samp_key = c->d_samp_key;
    sp.samp_counts = c->d_samp_counts;
    if (c->samp_cap) CU(cudaMemsetAsync(c->d_samp_n, 0, sizeof(unsigned long long), c->stream));
    sp.status = c->d_status;
    sp.quads_done = c->d_counters + 1;
    sp.prof = c->d_counters + 16;
    sp.debug = c->opts.debug;
    // debug 16: exact score for every quad.  K2: fp32 Stirling filter; chi-square: fp32 upper bound on X^2
    // (both phenotypes non-empty); MI: fp32 upper bound on M*I
    sp.use_filter = (sp.debug & 16) ? 0
                    : c->opts.objective == EPI4_OBJ_K2 ? 1
                    : (c->opts.objective == EPI4_OBJ_CHI2 && c->np[0] > 0 && c->np[1] > 0) ? 2
                    : c->opts.objective == EPI4_OBJ_MI ? 3 : 0;

    c->stats.launches = 0;
    CU(cudaEventRecord(c->ev[2], c->stream));
    int64_t acc = 0;
    int32_t slab_r = -1, slab_x = -1;
    for (const SearchPlan::Group& gr : pl.groups) {
        const int64_t gn = gr.e - gr.b, gtiles = pl.prefix[(size_t)gr.e - 1];
        if (gtiles == 0) continue;
        if (c->t3_windowed) {
            if (gr.wr != slab_r) {            // FIRST(R) into T3
                if (int r = build_t3_tc(c, c->T3, gr.wr * EPI4_WP, &c->stats.launches)) return r;
                slab_r = gr.wr;
                if (slab_x == slab_r) slab_x = -1;
            }
            if (gr.xr != gr.wr && gr.xr != slab_x) {   // FIRST(X) into T3x
                if (int r = build_t3_tc(c, c->T3x, gr.xr * EPI4_WP, &c->stats.launches)) return r;
                slab_x = gr.xr;
            }
            sp.d.t3_win = 1;
            sp.d.t3_w0 = gr.wr * EPI4_WP;
            sp.d.t3_x0 = gr.xr * EPI4_WP;
            sp.d.T3 = c->T3;
            sp.d.T3x = gr.xr == gr.wr ? c->T3 : c->T3x;
        }
        sp.units = c->d_units + gr.b;
        sp.prefix = c->d_prefix + gr.b;
        sp.nunits = gn;
        if (c->opts.pipe == EPI4_PIPE_LOP3) {
            sp.ntiles = gtiles;
            sp.tile_info = nullptr;
            CU(launch_quad_lop3(sp, grid, c->stream, &c->stats.launches));
        } else {
            // tiles in chunks of at most tile_chunk (bounded tile-table memory), one persistent launch each
            for (int64_t t0 = 0; t0 < gtiles; t0 += c->tile_chunk) {
                const int64_t t1 = std::min(gtiles, t0 + c->tile_chunk);
                const bool whole = pl.groups.size() == 1 && t0 == 0 && t1 == gtiles;
                if (!(whole && pl.table_cached)) {
                    CU(launch_tile_table(sp, t0, t1, c->d_tiles, c->stream, &c->stats.launches));
                    c->plan.table_cached = whole;
                }
                sp.tile_info = c->d_tiles;
                sp.ntiles = t1 - t0;
                CU(launch_quad_tc(sp, grid, c->stream, &c->stats.launches));
            }
        }
        acc += gtiles;
    }
    CU(cudaEventRecord(c->ev[3], c->stream));
    CU(launch_merge(sp, grid, c->d_out_k2, c->d_out_idx, c->d_out_n, c->stream, &c->stats.launches));
    int32_t nout = 0;
    unsigned long long ctr[32] = {0};
    CU(cudaMemcpyAsync(&nout, c->d_out_n, sizeof nout, cudaMemcpyDeviceToHost, c->stream));
    CU(cudaMemcpyAsync(quads_out, c->d_out_idx, (size_t)top_k * sizeof(uint64_t), cudaMemcpyDeviceToHost, c->stream));
    CU(cudaMemcpyAsync(k2_out, c->d_out_k2, (size_t)top_k * sizeof(double), cudaMemcpyDeviceToHost, c->stream));
    CU(cudaMemcpyAsync(ctr, c->d_counters, sizeof ctr, cudaMemcpyDeviceToHost, c->stream));
    CU(cudaEventRecord(c->ev[4], c->stream));
    CU(cudaStreamSynchronize(c->stream));
    float ms = 0;
    CU(cudaEventElapsedTime(&ms, c->ev[2], c->ev[3]));
    c->stats.ms_quad = ms;
    CU(cudaEventElapsedTime(&ms, c->ev[3], c->ev[4]));
    c->stats.ms_merge = ms;
    c->stats.quads = (int64_t)ctr[1];
    for (int i = 0; i < 8; ++i) c->stats.prof[i] = (double)ctr[16 + i];
    c->stats.tiles = acc / G;
    // MACs the contraction executes: 256 (w, a) rows (a 128-SNP w-range) x 8 YR columns per unit tile and
    // sample; the tensor-core operands run over whole steps (tc_chunks(yr) fp4 chunks of 256 samples,
    // zero-padded), the CUDA-core kernel over 128-sample chunks
    const double ksamples = c->opts.pipe == EPI4_PIPE_LOP3
                                ? (double)(c->nchunks[0] + c->nchunks[1]) * EPI4_CHUNK_SAMPLES
                                : (double)(tc_steps(sp.d.nchunks4[0], c->tc_yr) + tc_steps(sp.d.nchunks4[1], c->tc_yr)) * 256.0 *
                                      tc_chunks(c->tc_yr);
    c->stats.executed_macs = (double)(acc / G) * 256.0 * 8.0 * YR * ksamples;
    c->stats.tile_n = c->opts.pipe == EPI4_PIPE_LOP3 ? 0 : 8 * YR;
    *n_out = nout;
    return 0;
}

int epi4_search3(epi4_ctx* c, int32_t top_k, uint64_t* triples_out, double* k2_out, int32_t* n_out) {
    NvtxRange nvtx_range("epi4_search3");
    if (!c) return fail(EPI4_EINVAL, "ctx is NULL");
    if (!c->loaded) return fail(EPI4_ESTATE, "search before any load");
    if (c->opts.pipe != EPI4_PIPE_TC) return fail(EPI4_EINVAL, "the third-order search runs on the tensor-core pipe");
    if (c->n < 3) return fail(EPI4_EINVAL, "N=%d < 3", c->n);
    if (top_k < 1 || top_k > EPI4_MAX_TOPK) return fail(EPI4_EINVAL, "top_k=%d outside [1, %d]", top_k, EPI4_MAX_TOPK);
    if (!triples_out || !k2_out || !n_out) return fail(EPI4_EINVAL, "NULL output pointer");
    CU(cudaSetDevice(c->device));
    // this rank's units (the 4-way plan: w-range x second SNP) with z = the all-ones SNP n: each triple
    // w < x < y once across ranks
    std::vector<PlanEntry> plan = plan_rank(c->n, c->opts.rank, c->opts.world);
    std::vector<uint64_t>& tiles = c->host_tiles;
    tiles.clear();
    auto add = [&](int32_t wr, int32_t x) {
        for (int32_t y0 = x + 1; y0 <= c->n - 1; y0 += c->tc_yr)
            tiles.push_back((uint64_t)(uint16_t)wr | ((uint64_t)(uint16_t)x << 16) | ((uint64_t)(uint16_t)y0 << 32) |
                            ((uint64_t)(uint16_t)c->n << 48));
    };
    for (const PlanEntry& pe : plan) add(pe.u.wr, pe.u.x);
    // the 4-way plan has no units with x = n - 2 (no room for z); their triples (w, n - 2, n - 1) go to rank 0
    if (c->opts.rank == 0)
        for (int32_t wr = 0; wr * EPI4_WP < c->n - 2; ++wr) add(wr, c->n - 2);
    int32_t grid = c->opts.grid > 0 ? c->opts.grid : c->sm_count;
    grid = std::max(2, grid / 2 * 2);
    if (int r = ensure_lists(c, grid, top_k)) return r;
    CU(cudaMemsetAsync(c->d_list_cnt, 0, (size_t)grid * sizeof(int32_t), c->stream));
    CU(cudaMemsetAsync(c->d_counters, 0, 32 * sizeof(unsigned long long), c->stream));
    SearchParams sp{};
    sp.d = devdata(c);
    sp.yr = c->tc_yr;
    sp.t3_slab_w0 = -1;
    sp.search3 = 1;
    sp.topk = top_k;
    c->plan.table_cached = false;             // d_tiles is reused below
    sp.list_k2 = c->d_list_k2;
    sp.list_idx = c->d_list_idx;
    sp.list_cnt = c->d_list_cnt;
    sp.status = c->d_status;
    sp.quads_done = c->d_counters + 1;
    sp.prof = c->d_counters + 16;
    c->stats.launches = 0;
    CU(cudaEventRecord(c->ev[2], c->stream));
    if (!tiles.empty()) {
        CU(grow(c->d_tiles, c->cap_tiles, tiles.size() * sizeof(uint64_t)));
        CU(cudaMemcpyAsync(c->d_tiles, tiles.data(), tiles.size() * sizeof(uint64_t), cudaMemcpyHostToDevice,
                           c->stream));
        sp.tile_info = c->d_tiles;
        sp.ntiles = (int64_t)tiles.size();
        CU(launch_quad_tc(sp, grid, c->stream, &c->stats.launches));
    }
    CU(cudaEventRecord(c->ev[3], c->stream));
    CU(launch_merge(sp, grid, c->d_out_k2, c->d_out_idx, c->d_out_n, c->stream, &c->stats.launches));
    int32_t nout = 0;
    unsigned long long ctr[32] = {0};
    CU(cudaMemcpyAsync(&nout, c->d_out_n, sizeof nout, cudaMemcpyDeviceToHost, c->stream));
    CU(cudaMemcpyAsync(triples_out, c->d_out_idx, (size_t)top_k * sizeof(uint64_t), cudaMemcpyDeviceToHost, c->stream));
    CU(cudaMemcpyAsync(k2_out, c->d_out_k2, (size_t)top_k * sizeof(double), cudaMemcpyDeviceToHost, c->stream));
    CU(cudaMemcpyAsync(ctr, c->d_counters, sizeof ctr, cudaMemcpyDeviceToHost, c->stream));
    CU(cudaStreamSynchronize(c->stream));   // also keeps the host tile list alive for the copy
    float ms = 0;
    CU(cudaEventElapsedTime(&ms, c->ev[2], c->ev[3]));
    c->stats.ms_quad = ms;
    c->stats.quads = (int64_t)ctr[1];
    c->stats.tiles = (int64_t)tiles.size();
    *n_out = nout;
    return 0;
}

int epi4_search(epi4_ctx* c, int32_t top_k, uint64_t* quads_out, double* k2_out, int32_t* n_out) {
    return epi4_search_units(c, 0, -1, top_k, quads_out, k2_out, n_out);
}

int epi4_tables(epi4_ctx* c, const uint64_t* quads, int64_t n, uint32_t* counts_out) {
    if (!c) return fail(EPI4_EINVAL, "ctx is NULL");
    if (!c->loaded) return fail(EPI4_ESTATE, "tables before any load");
    if (c->t3_pending) return fail(EPI4_ESTATE, "sharded T3 incomplete: all-gather the shares, then epi4_t3_ready");
    if (c->t3_windowed) return fail(EPI4_ESTATE, "epi4_tables needs the resident 3-way table (windowed T3 in use)");
    if (n < 0 || (n > 0 && (!quads || !counts_out))) return fail(EPI4_EINVAL, "bad quads/counts arguments");
    if (n == 0) return 0;
    CU(cudaSetDevice(c->device));
    uint64_t* dq = nullptr;
    uint32_t* dc = nullptr;
    CU(cudaMalloc(&dq, (size_t)n * sizeof(uint64_t)));
    cudaError_t e = cudaMalloc(&dc, (size_t)n * 162 * sizeof(uint32_t));
    if (e == cudaSuccess) e = cudaMemcpyAsync(dq, quads, (size_t)n * sizeof(uint64_t), cudaMemcpyHostToDevice, c->stream);
    if (e == cudaSuccess) e = cudaMemsetAsync(c->d_status, 0, sizeof(unsigned int), c->stream);
    if (e == cudaSuccess) e = launch_tables(devdata(c), dq, n, dc, c->d_status, c->stream, nullptr);
    unsigned int st = 0;
    if (e == cudaSuccess)
        e = cudaMemcpyAsync(counts_out, dc, (size_t)n * 162 * sizeof(uint32_t), cudaMemcpyDeviceToHost, c->stream);
    if (e == cudaSuccess) e = cudaMemcpyAsync(&st, c->d_status, sizeof st, cudaMemcpyDeviceToHost, c->stream);
    if (e == cudaSuccess) e = cudaStreamSynchronize(c->stream);
    cudaFree(dq);
    if (dc) cudaFree(dc);
    CU(e);
    if (st) return fail(EPI4_EINVAL, "a quad has repeated SNPs or an SNP index >= N");
    return 0;
}

int epi4_get_stats(epi4_ctx* c, epi4_stats* out) {
    if (!c || !out) return fail(EPI4_EINVAL, "NULL argument");
    *out = c->stats;
    return 0;
}

}  // extern "C"
