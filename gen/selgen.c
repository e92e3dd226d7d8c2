/*
 * selgen.c -- seeded synthetic inputs for the five BASELINE.json configs.
 * INPUT DATA ONLY (see selgen.h): no counting, no model, no decision.
 *
 * Shapes follow the paper's Polybench list (§IV.E: GEMM, MVT, 3MM,
 * 2MM, ATAX, BICG, 2DCONV, 3DCONV, COVAR, GESUMMV, SYR2K, SYRK, CORR) split
 * into 24 parallel sub-kernels (SURVEY.md §8(d) shape table).  Sizes are
 * Polybench 4.2 MEDIUM (c2), 2^24-iteration parallel loops with inner trips
 * of 4 (c4), or the index-derived N of the c5 sweep.  The synthetic CPU cost
 * uses the form of the paper's Fig. 3 with the Table II constants
 * as a stand-in for the LLVM-MCA-derived cost the
 * paper supplies; it is an input of the hot path, not part of it.
 */
#include "selgen.h"
#include <string.h>

#define GOLDEN 0x9E3779B97F4A7C15ULL
#define SEED0 0x5E1EC7ULL
#define BASE0 0x10000000LL            /* 256 MiB: first array */
#define ARR_SPACING (1LL << 52)       /* arrays never overlap, all addresses < 2^55 */

uint64_t selgen_rng(uint64_t seed, uint64_t i) {
    uint64_t z = seed ^ (i * GOLDEN);
    z += GOLDEN;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
    return z ^ (z >> 31);
}

/* ---------------------------------------------------------------- shapes */
/* Loop variables: v0 = the parallel loop, v1, v2 = inner loops (v1 outer).
 * Each loop ranges over [0, size(sym) - sub).  Array dims are symbols.
 * An index expression is  c0*v0 + c1*v1 + c2*v2 + k  (k = stencil offset). */
typedef struct { int8_t arr, depth, store; int8_t idx[3][4]; } sh_access;
typedef struct { int8_t ndims, dim[3], role; } sh_array;   /* role: 1 read, 2 write, 3 both */
typedef struct {
    const char* name;
    int8_t n_inner;                  /* 1 or 2 inner loops */
    int8_t loopsym[3], loopsub[3];
    int16_t medium[4];               /* Polybench 4.2 MEDIUM symbol sizes */
    int8_t n_arr; sh_array arr[4];
    int8_t n_acc; sh_access acc[12];
    int8_t collapse_ok;              /* perfectly nested: collapse(2) variant exists */
} shape;

#define I(a,b,c,k) {a,b,c,k}
#define Z I(0,0,0,0)
#define A1(arr,d,st,e0) {arr,d,st,{e0,Z,Z}}
#define A2(arr,d,st,e0,e1) {arr,d,st,{e0,e1,Z}}
#define A3(arr,d,st,e0,e1,e2) {arr,d,st,{e0,e1,e2}}
#define V0 I(1,0,0,0)
#define V1 I(0,1,0,0)
#define V2 I(0,0,1,0)

static const shape SHAPES[24] = {
  /* gemm: C[i][j] += A[i][k]*B[k][j]; NI,NJ,NK */
  {"gemm", 2, {0,1,2},{0,0,0}, {200,220,240,0}, 3,
   {{2,{0,2},1},{2,{2,1},1},{2,{0,1},3}}, 3,
   {A2(0,2,0,V0,V2), A2(1,2,0,V2,V1), A2(2,2,1,V0,V1)}, 1},
  /* 2mm.1: tmp[i][j] += A[i][k]*B[k][j]; NI,NJ,NK */
  {"2mm.1", 2, {0,1,2},{0,0,0}, {180,190,210,0}, 3,
   {{2,{0,2},1},{2,{2,1},1},{2,{0,1},2}}, 3,
   {A2(0,2,0,V0,V2), A2(1,2,0,V2,V1), A2(2,2,1,V0,V1)}, 0},
  /* 2mm.2: D[i][j] += tmp[i][k]*C[k][j]; NI,NL,NJ */
  {"2mm.2", 2, {0,1,2},{0,0,0}, {180,220,190,0}, 3,
   {{2,{0,2},1},{2,{2,1},1},{2,{0,1},3}}, 3,
   {A2(0,2,0,V0,V2), A2(1,2,0,V2,V1), A2(2,2,1,V0,V1)}, 0},
  /* 3mm.1: E = A*B; NI,NJ,NK */
  {"3mm.1", 2, {0,1,2},{0,0,0}, {180,190,200,0}, 3,
   {{2,{0,2},1},{2,{2,1},1},{2,{0,1},2}}, 3,
   {A2(0,2,0,V0,V2), A2(1,2,0,V2,V1), A2(2,2,1,V0,V1)}, 0},
  /* 3mm.2: F = C*D; NJ,NL,NM */
  {"3mm.2", 2, {0,1,2},{0,0,0}, {190,210,220,0}, 3,
   {{2,{0,2},1},{2,{2,1},1},{2,{0,1},2}}, 3,
   {A2(0,2,0,V0,V2), A2(1,2,0,V2,V1), A2(2,2,1,V0,V1)}, 0},
  /* 3mm.3: G = E*F; NI,NL,NJ */
  {"3mm.3", 2, {0,1,2},{0,0,0}, {180,210,190,0}, 3,
   {{2,{0,2},1},{2,{2,1},1},{2,{0,1},2}}, 3,
   {A2(0,2,0,V0,V2), A2(1,2,0,V2,V1), A2(2,2,1,V0,V1)}, 0},
  /* atax.1: tmp[i] = 0; tmp[i] += A[i][j]*x[j]; M,N */
  {"atax.1", 1, {0,1,0},{0,0,0}, {390,410,0,0}, 3,
   {{2,{0,1},1},{1,{1},1},{1,{0},3}}, 4,
   {A1(2,0,1,V0), A2(0,1,0,V0,V1), A1(1,1,0,V1), A1(2,1,1,V0)}, 0},
  /* atax.2: y[j] = 0; y[j] += A[i][j]*tmp[i]  (parallel j); j<N, i<M */
  {"atax.2", 1, {1,0,0},{0,0,0}, {390,410,0,0}, 3,
   {{2,{0,1},1},{1,{0},1},{1,{1},3}}, 4,
   {A1(2,0,1,V0), A2(0,1,0,V1,V0), A1(1,1,0,V1), A1(2,1,1,V0)}, 0},
  /* bicg.1: s[j] = 0; s[j] += r[i]*A[i][j]  (parallel j); j<M, i<N */
  {"bicg.1", 1, {0,1,0},{0,0,0}, {390,410,0,0}, 3,
   {{2,{1,0},1},{1,{1},1},{1,{0},3}}, 4,
   {A1(2,0,1,V0), A2(0,1,0,V1,V0), A1(1,1,0,V1), A1(2,1,1,V0)}, 0},
  /* bicg.2: q[i] = 0; q[i] += A[i][j]*p[j]; i<N, j<M */
  {"bicg.2", 1, {1,0,0},{0,0,0}, {390,410,0,0}, 3,
   {{2,{1,0},1},{1,{0},1},{1,{1},3}}, 4,
   {A1(2,0,1,V0), A2(0,1,0,V0,V1), A1(1,1,0,V1), A1(2,1,1,V0)}, 0},
  /* mvt.1: x1[i] += A[i][j]*y1[j]; N */
  {"mvt.1", 1, {0,0,0},{0,0,0}, {400,0,0,0}, 3,
   {{2,{0,0},1},{1,{0},1},{1,{0},3}}, 3,
   {A2(0,1,0,V0,V1), A1(1,1,0,V1), A1(2,1,1,V0)}, 0},
  /* mvt.2: x2[i] += A[j][i]*y2[j]; N */
  {"mvt.2", 1, {0,0,0},{0,0,0}, {400,0,0,0}, 3,
   {{2,{0,0},1},{1,{0},1},{1,{0},3}}, 3,
   {A2(0,1,0,V1,V0), A1(1,1,0,V1), A1(2,1,1,V0)}, 0},
  /* gesummv: tmp[i] += A[i][j]*x[j]; y[i] += B[i][j]*x[j]; N */
  {"gesummv", 1, {0,0,0},{0,0,0}, {250,0,0,0}, 4,
   {{2,{0,0},1},{2,{0,0},1},{1,{0},1},{1,{0},3}}, 5,
   {A2(0,1,0,V0,V1), A2(1,1,0,V0,V1), A1(2,1,0,V1), A1(3,1,1,V0), A1(3,1,1,V0)}, 0},
  /* syrk: C[i][j] += A[i][k]*A[j][k]; N (i, j), M (k) -- triangle as rectangle */
  {"syrk", 2, {0,0,1},{0,0,0}, {240,200,0,0}, 2,
   {{2,{0,1},1},{2,{0,0},3}}, 3,
   {A2(0,2,0,V0,V2), A2(0,2,0,V1,V2), A2(1,2,1,V0,V1)}, 0},
  /* syr2k: C[i][j] += A[j][k]*B[i][k] + B[j][k]*A[i][k]; N, M */
  {"syr2k", 2, {0,0,1},{0,0,0}, {240,200,0,0}, 3,
   {{2,{0,1},1},{2,{0,1},1},{2,{0,0},3}}, 5,
   {A2(0,2,0,V0,V2), A2(1,2,0,V0,V2), A2(0,2,0,V1,V2), A2(1,2,0,V1,V2), A2(2,2,1,V0,V1)}, 0},
  /* cov.mean: mean[j] = 0; mean[j] += data[i][j]  (parallel j); M (j), N (i) */
  {"cov.mean", 1, {0,1,0},{0,0,0}, {240,260,0,0}, 2,
   {{2,{1,0},1},{1,{0},3}}, 3,
   {A1(1,0,1,V0), A2(0,1,0,V1,V0), A1(1,1,1,V0)}, 0},
  /* cov.reduce: data[i][j] -= mean[j]; i<N, j<M */
  {"cov.reduce", 1, {1,0,0},{0,0,0}, {240,260,0,0}, 2,
   {{2,{1,0},3},{1,{0},1}}, 2,
   {A2(0,1,1,V0,V1), A1(1,1,0,V1)}, 0},
  /* cov.covar: cov[i][j] += data[k][i]*data[k][j]; M (i, j), N (k) */
  {"cov.covar", 2, {0,0,1},{0,0,0}, {240,260,0,0}, 2,
   {{2,{1,0},1},{2,{0,0},3}}, 3,
   {A2(0,2,0,V2,V0), A2(0,2,0,V2,V1), A2(1,2,1,V0,V1)}, 0},
  /* corr.mean: mean[j] += data[i][j]  (parallel j) */
  {"corr.mean", 1, {0,1,0},{0,0,0}, {240,260,0,0}, 2,
   {{2,{1,0},1},{1,{0},3}}, 3,
   {A1(1,0,1,V0), A2(0,1,0,V1,V0), A1(1,1,1,V0)}, 0},
  /* corr.std: std[j] += (data[i][j]-mean[j])^2  (parallel j) */
  {"corr.std", 1, {0,1,0},{0,0,0}, {240,260,0,0}, 3,
   {{2,{1,0},1},{1,{0},1},{1,{0},3}}, 3,
   {A2(0,1,0,V1,V0), A1(1,1,0,V0), A1(2,1,1,V0)}, 0},
  /* corr.reduce: data[i][j] = (data[i][j]-mean[j])/std[j]; i<N, j<M */
  {"corr.reduce", 1, {1,0,0},{0,0,0}, {240,260,0,0}, 3,
   {{2,{1,0},3},{1,{0},1},{1,{0},1}}, 3,
   {A2(0,1,1,V0,V1), A1(1,1,0,V1), A1(2,1,0,V1)}, 0},
  /* corr.corr: corr[i][j] += data[k][i]*data[k][j]; i<M-1, j<M, k<N */
  {"corr.corr", 2, {0,0,1},{1,0,0}, {240,260,0,0}, 2,
   {{2,{1,0},1},{2,{0,0},3}}, 3,
   {A2(0,2,0,V2,V0), A2(0,2,0,V2,V1), A2(1,2,1,V0,V1)}, 0},
  /* 2DCONV (PolyBench/GPU): B[i+1][j+1] = sum_{di,dj in 0..2} c*A[i+di][j+dj] */
  {"2DCONV", 1, {0,1,0},{2,2,0}, {1100,1100,0,0}, 2,
   {{2,{0,1},1},{2,{0,1},2}}, 10,
   {A2(0,1,0,I(1,0,0,0),I(0,1,0,0)), A2(0,1,0,I(1,0,0,0),I(0,1,0,1)), A2(0,1,0,I(1,0,0,0),I(0,1,0,2)),
    A2(0,1,0,I(1,0,0,1),I(0,1,0,0)), A2(0,1,0,I(1,0,0,1),I(0,1,0,1)), A2(0,1,0,I(1,0,0,1),I(0,1,0,2)),
    A2(0,1,0,I(1,0,0,2),I(0,1,0,0)), A2(0,1,0,I(1,0,0,2),I(0,1,0,1)), A2(0,1,0,I(1,0,0,2),I(0,1,0,2)),
    A2(1,1,1,I(1,0,0,1),I(0,1,0,1))}, 1},
  /* 3DCONV (PolyBench/GPU style): B[i+1][j+1][k+1] = 11-point stencil of A */
  {"3DCONV", 2, {0,1,2},{2,2,2}, {128,128,128,0}, 2,
   {{3,{0,1,2},1},{3,{0,1,2},2}}, 12,
   {A3(0,2,0,I(1,0,0,0),I(0,1,0,0),I(0,0,1,0)), A3(0,2,0,I(1,0,0,2),I(0,1,0,0),I(0,0,1,0)),
    A3(0,2,0,I(1,0,0,1),I(0,1,0,0),I(0,0,1,1)), A3(0,2,0,I(1,0,0,1),I(0,1,0,1),I(0,0,1,1)),
    A3(0,2,0,I(1,0,0,1),I(0,1,0,2),I(0,0,1,1)), A3(0,2,0,I(1,0,0,0),I(0,1,0,0),I(0,0,1,2)),
    A3(0,2,0,I(1,0,0,2),I(0,1,0,0),I(0,0,1,2)), A3(0,2,0,I(1,0,0,0),I(0,1,0,1),I(0,0,1,2)),
    A3(0,2,0,I(1,0,0,2),I(0,1,0,1),I(0,0,1,2)), A3(0,2,0,I(1,0,0,0),I(0,1,0,2),I(0,0,1,2)),
    A3(0,2,0,I(1,0,0,2),I(0,1,0,2),I(0,0,1,2)),
    A3(1,2,1,I(1,0,0,1),I(0,1,0,1),I(0,0,1,1))}, 1},
};

int selgen_num_shapes(void) { return 24; }
const char* selgen_shape_name(int s) { return (s >= 0 && s < 24) ? SHAPES[s].name : 0; }

/* ------------------------------------------------------- device / launch */
int selgen_device_sets(gen_device_params* o) {
    /* Table III names the parameters but its values were lost;
     * these are builder-chosen public/vendor figures (R23).  The
     * last four fields are NEXT row f4's (F4c, F4d): register
     * allocation unit 256 registers per warp, warp allocation granularity 4,
     * shared-memory allocation unit 256 B (the CUDA occupancy calculator's
     * values for these generations), and the transaction unit -- 128 B lines
     * (H&K) for K80 / P100 / V100 as in the paper, 32 B sectors for B200. */
    const gen_device_params d[4] = {
        /* K80, one GK210 */
        {13, 64, 2048, 16, 131072, 114688, 0.875e9, 240.48e9, 12.0e9, 5.0e-6, 440.0, 4.0, 12.0, 4.0, 256, 4, 256, 0},
        /* P100 SXM2 */
        {56, 64, 2048, 32, 65536, 65536, 1.480e9, 732.0e9, 32.0e9, 4.0e-6, 500.0, 4.0, 10.0, 2.0, 256, 4, 256, 0},
        /* V100 SXM2 (AC922, NVLink 2: 3 bricks x 25 GB/s) */
        {80, 64, 2048, 32, 65536, 98304, 1.530e9, 900.0e9, 75.0e9, 4.0e-6, 440.0, 4.0, 10.0, 2.0, 256, 4, 256, 0},
        /* B200 */
        {148, 64, 2048, 32, 65536, 233472, 1.965e9, 7.7e12, 55.0e9, 3.0e-6, 600.0, 4.0, 8.0, 2.0, 256, 4, 256, 1},
    };
    memcpy(o, d, sizeof d);
    return 4;
}

int selgen_launches(int cfg, gen_launch* o) {
    switch (cfg) {
    case SELGEN_C1: o[0] = (gen_launch){256, 65535, 32, 0}; return 1;
    case SELGEN_C2: o[0] = (gen_launch){128, 65535, 32, 0}; return 1;
    case SELGEN_C3: o[0] = (gen_launch){256, 65535, 32, 0}; return 1;
    case SELGEN_C4: case SELGEN_C5: {
        static const uint32_t Bs[4] = {48, 128, 200, 1024};
        for (int i = 0; i < 8; i++)
            o[i] = (gen_launch){Bs[i >> 1], (i & 1) ? 65535u : 160u, 32, 0};
        return 8;
    }
    default: return -1;
    }
}

uint64_t selgen_num_candidates(int cfg) {
    switch (cfg) {
    case SELGEN_C1: return 2;
    case SELGEN_C2: return 108;
    case SELGEN_C3: return 1000000;
    case SELGEN_C4: return 192;
    case SELGEN_C5: return 100000000ULL;
    default: return 0;
    }
}

/* ----------------------------------------------------------- nest build */
typedef struct {
    uint64_t symsz[4];     /* symbol sizes */
    uint64_t ext[3];       /* loop extents v0, v1, v2 */
    int elem;
    int64_t arr_off[4];    /* per-array base offset in bytes */
    int collapse;
    int threads;           /* synthetic host thread count for cpu_cycles */
} nest_params;

static uint64_t ceil_div_u64(uint64_t a, uint64_t b) { return (a + b - 1) / b; }

/* Fills one nest and its accesses; returns the synthetic cpu_cycles. */
static double build_nest(const shape* sh, const nest_params* np, gen_nest* n,
                         gen_access* acc, uint32_t access_off) {
    memset(n, 0, sizeof *n);
    const int b = np->elem;
    int64_t rowstride[4][3];
    uint64_t arrbytes[4];
    for (int a = 0; a < sh->n_arr; a++) {
        const sh_array* ar = &sh->arr[a];
        int64_t s = 1;
        for (int d = ar->ndims - 1; d >= 0; d--) { rowstride[a][d] = s; s *= (int64_t)np->symsz[ar->dim[d]]; }
        arrbytes[a] = (uint64_t)s * (uint64_t)b;
    }
    if (np->collapse) {
        n->par_dims = 2; n->P0 = np->ext[0]; n->P1 = np->ext[1];
        n->depth = (uint8_t)(sh->n_inner - 1);
        n->trip[0] = (uint32_t)np->ext[2];
    } else {
        n->par_dims = 1; n->P0 = np->ext[0]; n->P1 = 1;
        n->depth = (uint8_t)sh->n_inner;
        n->trip[0] = (uint32_t)np->ext[1];
        if (sh->n_inner == 2) n->trip[1] = (uint32_t)np->ext[2];
    }
    n->access_off = access_off;
    n->n_access = (uint32_t)sh->n_acc;
    int per_depth[4] = {0, 0, 0, 0};
    for (int k = 0; k < sh->n_acc; k++) {
        const sh_access* sa = &sh->acc[k];
        const sh_array* ar = &sh->arr[sa->arr];
        int64_t cv[3] = {0, 0, 0}, koff = 0;
        for (int d = 0; d < ar->ndims; d++) {
            for (int v = 0; v < 3; v++) cv[v] += sa->idx[d][v] * rowstride[sa->arr][d];
            koff += sa->idx[d][3] * rowstride[sa->arr][d];
        }
        gen_access* g = &acc[k];
        memset(g, 0, sizeof *g);
        g->base = BASE0 + (int64_t)sa->arr * ARR_SPACING + np->arr_off[sa->arr] + koff * b;
        g->elem_bytes = (uint8_t)b;
        g->is_store = (uint8_t)sa->store;
        if (np->collapse) {
            g->c_par[0] = cv[0] * b; g->c_par[1] = cv[1] * b; g->c_inner[0] = cv[2] * b;
            g->depth = (uint8_t)(sa->depth - 1);
        } else {
            g->c_par[0] = cv[0] * b; g->c_inner[0] = cv[1] * b; g->c_inner[1] = cv[2] * b;
            g->depth = (uint8_t)sa->depth;
        }
        per_depth[g->depth]++;
    }
    /* Synthetic instruction loadout (stand-in for the static IR count of
     * P:L158-159): 2 compute instructions per access at that level plus
     * loop/index overhead. */
    for (int d = 0; d <= n->depth; d++) n->comp_insts[d] = 2.0 * per_depth[d] + (d == 0 ? 4.0 : 2.0);
    for (int a = 0; a < sh->n_arr; a++) {
        if (sh->arr[a].role & 1) n->bytes_h2d += arrbytes[a];
        if (sh->arr[a].role & 2) n->bytes_d2h += arrbytes[a];
    }
    /* Fig. 3 form with Table II constants: Par_Startup 3000 + static
     * schedule 10154 + chunk work + sync 4000. */
    uint64_t P = np->collapse ? np->ext[0] * np->ext[1] : np->ext[0];
    uint64_t inner = 1;
    for (int j = 0; j < sh->n_inner - (np->collapse ? 1 : 0); j++) inner *= np->collapse ? np->ext[2] : np->ext[1 + j];
    double mca_k = 2.0 + 0.5 * (double)sh->n_acc;
    return 3000.0 + 10154.0 + (double)ceil_div_u64(P, (uint64_t)np->threads) * (mca_k * (double)inner + 4.0) + 4000.0;
}

/* sizes of shape s in config cfg, with c5 parameter z */
static void shape_params(const shape* sh, int cfg, uint64_t z, int collapse, nest_params* np) {
    memset(np, 0, sizeof *np);
    np->collapse = collapse;
    np->threads = 160;
    if (cfg == SELGEN_C1) {                        /* GEMM N = 64, fp32 */
        for (int i = 0; i < 4; i++) np->symsz[i] = 64;
        np->elem = 4;
    } else if (cfg == SELGEN_C2) {                 /* Polybench MEDIUM, fp64 */
        for (int i = 0; i < 4; i++) np->symsz[i] = (uint64_t)sh->medium[i];
        np->elem = 8;
    } else if (cfg == SELGEN_C4) {                 /* parallel trip 2^24, inner trips 4 */
        for (int i = 0; i < 4; i++) np->symsz[i] = 4;
        np->elem = 8;
    } else {                                       /* c5 */
        uint64_t N = (sh->n_inner == 1) ? 16 + (z % 497) : 8 + (z % 57);
        for (int i = 0; i < 4; i++) np->symsz[i] = N;
        np->elem = (z % 2 == 0) ? 4 : 8;
        for (int a = 0; a < 4; a++)
            np->arr_off[a] = (int64_t)(((z / 497) + 7 * (uint64_t)a) % (uint64_t)(128 / np->elem)) * np->elem;
        np->threads = ((z / 2) % 2 == 0) ? 160 : 4;
    }
    if (cfg == SELGEN_C4) {
        /* the parallel loop's symbol is 2^24 (+sub); inner extents forced to 4 */
        int s0 = sh->loopsym[0];
        uint64_t maxsub = 0;
        for (int v = 0; v <= sh->n_inner; v++) if (sh->loopsym[v] == s0 && (uint64_t)sh->loopsub[v] > maxsub) maxsub = (uint64_t)sh->loopsub[v];
        np->symsz[s0] = (1ULL << 24) + maxsub;
        for (int v = 1; v <= sh->n_inner; v++) {
            int s = sh->loopsym[v];
            if (s != s0 && np->symsz[s] < 4 + (uint64_t)sh->loopsub[v]) np->symsz[s] = 4 + (uint64_t)sh->loopsub[v];
        }
        np->ext[0] = 1ULL << 24;
        for (int v = 1; v <= sh->n_inner; v++) np->ext[v] = 4;
    } else {
        for (int v = 0; v <= sh->n_inner; v++) np->ext[v] = np->symsz[sh->loopsym[v]] - (uint64_t)sh->loopsub[v];
    }
}

/* c2 nest list: 24 shapes, then collapse(2) variants of gemm, 2DCONV, 3DCONV */
static int c2_nest(int idx, int* collapse) {
    if (idx < 24) { *collapse = 0; return idx; }
    static const int cv[3] = {0, 22, 23};
    *collapse = 1;
    return cv[idx - 24];
}

int selgen_count(int cfg, uint64_t c0, uint64_t c1, uint64_t* n_nests, uint64_t* n_access) {
    uint64_t N = selgen_num_candidates(cfg);
    if (c0 > c1 || c1 > N) return -1;
    uint64_t nn = 0, na = 0;
    switch (cfg) {
    case SELGEN_C1: nn = 2; na = 6; break;
    case SELGEN_C2: for (int i = 0; i < 27; i++) { int col; nn++; na += (uint64_t)SHAPES[c2_nest(i, &col)].n_acc; } break;
    case SELGEN_C3: nn = c1 - c0; na = c1 - c0; break;
    case SELGEN_C4: nn = 24; for (int s = 0; s < 24; s++) na += (uint64_t)SHAPES[s].n_acc; break;
    case SELGEN_C5:
        if (c1 > c0) {
            uint64_t g0 = c0 / 32, g1 = (c1 - 1) / 32;   /* groups of 32 share a nest */
            nn = g1 - g0 + 1;
            for (uint64_t g = g0; g <= g1; g++) na += (uint64_t)SHAPES[g % 24].n_acc;
        }
        break;
    default: return -1;
    }
    *n_nests = nn; *n_access = na;
    return 0;
}

int selgen_fill(int cfg, uint64_t c0, uint64_t c1, gen_candidate* cands, gen_nest* nests, gen_access* acc) {
    uint64_t N = selgen_num_candidates(cfg);
    if (c0 > c1 || c1 > N) return -1;
    const double cpu_hz = 3.0e9;   /* Table II: CPU frequency 3 GHz */
    nest_params np;
    if (cfg == SELGEN_C1) {
        for (int v = 0; v < 2; v++) {
            shape_params(&SHAPES[0], cfg, 0, v, &np);
            double cyc = build_nest(&SHAPES[0], &np, &nests[v], &acc[3 * v], (uint32_t)(3 * v));
            nests[v].bytes_h2d = 3 * 64 * 64 * 4; nests[v].bytes_d2h = 64 * 64 * 4;
            if (v >= (int)c0 && v < (int)c1)
                cands[v - c0] = (gen_candidate){(uint32_t)v, 0, 2, cyc, cpu_hz};
        }
        return 0;
    }
    if (cfg == SELGEN_C2) {
        double cyc[27];
        uint32_t off = 0;
        for (int i = 0; i < 27; i++) {
            int col, s = c2_nest(i, &col);
            shape_params(&SHAPES[s], cfg, 0, col, &np);
            np.threads = (i & 1) ? 4 : 160;
            cyc[i] = build_nest(&SHAPES[s], &np, &nests[i], &acc[off], off);
            off += (uint32_t)SHAPES[s].n_acc;
        }
        for (uint64_t c = c0; c < c1; c++)
            cands[c - c0] = (gen_candidate){(uint32_t)(c / 4), 0, (uint16_t)(c % 4), cyc[c / 4], cpu_hz};
        return 0;
    }
    if (cfg == SELGEN_C3) {
        const uint64_t seed = SEED0 + 3;
        for (uint64_t c = c0; c < c1; c++) {
            uint64_t i = c, k = c - c0;
            int64_t s = 1 + (int64_t)(i % 64);
            int b = 4 << ((i / 64) % 2);
            int64_t o = (int64_t)b * (int64_t)((i / 128) % (uint64_t)(128 / b));
            uint64_t P = 1 + selgen_rng(seed, 2 * i) % 4096;
            int neg = (selgen_rng(seed, 2 * i + 1) % 100) == 0;
            gen_nest* n = &nests[k];
            memset(n, 0, sizeof *n);
            n->P0 = P; n->P1 = 1; n->par_dims = 1; n->depth = 0;
            n->trip[0] = n->trip[1] = n->trip[2] = 1;
            n->comp_insts[0] = 4.0;
            n->access_off = (uint32_t)k; n->n_access = 1;
            gen_access* g = &acc[k];
            memset(g, 0, sizeof *g);
            g->elem_bytes = (uint8_t)b; g->depth = 0; g->is_store = (uint8_t)(i & 1);
            int64_t span = (int64_t)(P - 1) * s * b;
            if (neg) { g->base = BASE0 + o + span; g->c_par[0] = -s * b; }
            else     { g->base = BASE0 + o;        g->c_par[0] = s * b; }
            uint64_t bytes = (uint64_t)span + (uint64_t)b;
            if (g->is_store) n->bytes_d2h = bytes; else n->bytes_h2d = bytes;
            int threads = ((i >> 1) & 1) ? 4 : 160;
            double cyc = 3000.0 + 10154.0 + (double)ceil_div_u64(P, (uint64_t)threads) * (2.5 + 4.0) + 4000.0;
            cands[k] = (gen_candidate){(uint32_t)k, 0, 2, cyc, cpu_hz};
        }
        return 0;
    }
    if (cfg == SELGEN_C4) {
        double cyc[24];
        uint32_t off = 0;
        for (int s = 0; s < 24; s++) {
            shape_params(&SHAPES[s], cfg, 0, 0, &np);
            cyc[s] = build_nest(&SHAPES[s], &np, &nests[s], &acc[off], off);
            off += (uint32_t)SHAPES[s].n_acc;
        }
        for (uint64_t c = c0; c < c1; c++)
            cands[c - c0] = (gen_candidate){(uint32_t)(c / 8), (uint16_t)(c % 8), 2, cyc[c / 8], cpu_hz};
        return 0;
    }
    if (cfg == SELGEN_C5) {
        if (c1 == c0) return 0;
        uint64_t g0 = c0 / 32, g1 = (c1 - 1) / 32;
        uint32_t off = 0;
        double cyc = 0.0;
        uint64_t c = c0;
        for (uint64_t g = g0; g <= g1; g++) {
            uint64_t z = g / 24;
            int s = (int)(g % 24);
            shape_params(&SHAPES[s], cfg, z, 0, &np);
            cyc = build_nest(&SHAPES[s], &np, &nests[g - g0], &acc[off], off);
            off += (uint32_t)SHAPES[s].n_acc;
            uint64_t end = (g + 1) * 32 < c1 ? (g + 1) * 32 : c1;
            for (; c < end; c++)
                cands[c - c0] = (gen_candidate){(uint32_t)(g - g0), (uint16_t)((c / 4) % 8), (uint16_t)(c % 4), cyc, cpu_hz};
        }
        return 0;
    }
    return -1;
}

/* Candidates idx[0..m) of an index-addressable config (c3, c5), each with
 * its own copy of the nest it references (nests[i], accesses from a running
 * offset).  Used to draw bounded, strided samples of a sweep. */
int selgen_count_indices(int cfg, const uint64_t* idx, uint64_t m, uint64_t* n_access) {
    uint64_t na = 0;
    for (uint64_t i = 0; i < m; i++) {
        if (idx[i] >= selgen_num_candidates(cfg)) return -1;
        if (cfg == SELGEN_C5) na += (uint64_t)SHAPES[(idx[i] / 32) % 24].n_acc;
        else if (cfg == SELGEN_C3) na += 1;
        else return -1;
    }
    *n_access = na;
    return 0;
}

int selgen_fill_indices(int cfg, const uint64_t* idx, uint64_t m, gen_candidate* cands, gen_nest* nests,
                        gen_access* acc) {
    uint64_t off = 0;
    for (uint64_t i = 0; i < m; i++) {
        uint64_t c = idx[i], na = 0, nn = 0;
        if (selgen_count(cfg, c, c + 1, &nn, &na) != 0) return -1;
        if (selgen_fill(cfg, c, c + 1, &cands[i], &nests[i], &acc[off]) != 0) return -1;
        nests[i].access_off = (uint32_t)off;
        cands[i].nest_id = (uint32_t)i;
        off += na;
    }
    return 0;
}

/* ------------------------------------------------------------ CPU inputs */
/* Inputs of the NEXT-row f1 CPU model (Liao-Chapman, Fig. 3): the LLVM-MCA
 * stand-in cycles per parallel iteration (mca_k x product of inner trips,
 * the same synthetic loadout that produced cpu_cycles above) and the host
 * thread count.  With a TLB term of zero the modelled cost equals the
 * supplied cpu_cycles of the candidate. */
static void cand_cpu(int cfg, uint64_t c, double* mca, uint32_t* threads) {
    nest_params np;
    const shape* sh;
    int col = 0;
    if (cfg == SELGEN_C3) {
        *mca = 2.5;
        *threads = ((c >> 1) & 1) ? 4u : 160u;
        return;
    }
    if (cfg == SELGEN_C1) { sh = &SHAPES[0]; col = (int)c; shape_params(sh, cfg, 0, col, &np); }
    else if (cfg == SELGEN_C2) {
        int idx = (int)(c / 4), s = c2_nest(idx, &col);
        sh = &SHAPES[s];
        shape_params(sh, cfg, 0, col, &np);
        np.threads = (idx & 1) ? 4 : 160;
    } else if (cfg == SELGEN_C4) { sh = &SHAPES[c / 8]; shape_params(sh, cfg, 0, 0, &np); }
    else { uint64_t g = c / 32; sh = &SHAPES[g % 24]; shape_params(sh, cfg, g / 24, 0, &np); }
    uint64_t inner = 1;
    for (int j = 0; j < sh->n_inner - (col ? 1 : 0); j++) inner *= col ? np.ext[2] : np.ext[1 + j];
    *mca = (2.0 + 0.5 * (double)sh->n_acc) * (double)inner;
    *threads = (uint32_t)np.threads;
}

int selgen_cpu_inputs(int cfg, uint64_t c0, uint64_t c1, gen_cpu_input* out) {
    if (c0 > c1 || c1 > selgen_num_candidates(cfg)) return -1;
    for (uint64_t c = c0; c < c1; c++) {
        out[c - c0].mca_cycles_per_iter = 0.0;
        out[c - c0]._pad = 0;
        cand_cpu(cfg, c, &out[c - c0].mca_cycles_per_iter, &out[c - c0].threads);
    }
    return 0;
}

void selgen_cpu_params(gen_cpu_params* p) {
    /* Table II plus the 64 KiB base page of Linux on POWER9
     * (the page size is not in the paper; reading F1c). */
    p->cpu_hz = 3.0e9;
    p->tlb_entries = 1024.0;
    p->tlb_miss_cycles = 14.0;
    p->loop_overhead_cycles = 4.0;
    p->schedule_static_cycles = 10154.0;
    p->sync_cycles = 4000.0;
    p->startup_cycles = 3000.0;
    p->page_bytes = 65536.0;
}

/* ------------------------------------------------------ symbolic accesses */
/* NEXT row f2 inputs: the accesses of every shape as IPDA-style symbolic
 * expressions: each byte coefficient is a sum of terms
 * k * v[s0] * v[s1] * v[s2] over a per-nest-instance symbol frame
 *   frame = [elem, size(sym0..sym3), array_offset(0..3)]           (9 values)
 * Binding the frame reproduces exactly the concrete accesses selgen_fill
 * writes.  Symbolic table index: (2 * shape + collapse) * 12 + access. */
#define FR_ELEM 0
#define FR_SIZE 1
#define FR_OFF 5
#define SYM_ONE 0xFFFFu

static uint32_t sym_term(gen_sym_term* terms, uint32_t* nt, int64_t k, uint16_t s0, uint16_t s1, uint16_t s2) {
    if (terms) { terms[*nt].k = k; terms[*nt].sym[0] = s0; terms[*nt].sym[1] = s1; terms[*nt].sym[2] = s2; terms[*nt]._pad = 0; }
    return (*nt)++;
}

int selgen_sym_tables(gen_sym_access* sym, gen_sym_term* terms, uint32_t* n_sym, uint32_t* n_terms) {
    uint32_t nt = 0;
    for (int s = 0; s < 24; s++) {
        const shape* sh = &SHAPES[s];
        for (int col = 0; col < 2; col++) {
            for (int k = 0; k < 12; k++) {
                gen_sym_access* g = sym ? &sym[(2 * s + col) * 12 + k] : 0;
                if (g) memset(g, 0, sizeof *g);
                if (k >= sh->n_acc || (col && !sh->collapse_ok)) continue;
                const sh_access* sa = &sh->acc[k];
                const sh_array* ar = &sh->arr[sa->arr];
                /* coefficient slots: 0 base, 1 c_par[0], 2 c_par[1], 3..5 c_inner[0..2] */
                int slot_of_var[3];
                if (col) { slot_of_var[0] = 1; slot_of_var[1] = 2; slot_of_var[2] = 3; }
                else { slot_of_var[0] = 1; slot_of_var[1] = 3; slot_of_var[2] = 4; }
                for (int slot = 0; slot < 6; slot++) {
                    uint32_t first = nt, cnt = 0;
                    if (slot == 0) {
                        sym_term(terms, &nt, BASE0 + (int64_t)sa->arr * ARR_SPACING, SYM_ONE, SYM_ONE, SYM_ONE); cnt++;
                        sym_term(terms, &nt, 1, (uint16_t)(FR_OFF + sa->arr), SYM_ONE, SYM_ONE); cnt++;
                    }
                    for (int d = 0; d < ar->ndims; d++) {
                        int64_t kk = 0;
                        if (slot == 0) kk = sa->idx[d][3];
                        else for (int v = 0; v < 3; v++) if (slot_of_var[v] == slot) kk += sa->idx[d][v];
                        if (kk == 0) continue;
                        /* row stride of dim d: product of the later dims' sizes */
                        uint16_t f[2] = {SYM_ONE, SYM_ONE};
                        int nf = 0;
                        for (int d2 = d + 1; d2 < ar->ndims; d2++) f[nf++] = (uint16_t)(FR_SIZE + ar->dim[d2]);
                        sym_term(terms, &nt, kk, FR_ELEM, f[0], f[1]);
                        cnt++;
                    }
                    if (g) { g->term_off[slot] = first; g->n_terms[slot] = (uint8_t)cnt; }
                }
                if (g) {
                    g->elem_sym = FR_ELEM;
                    g->elem_bytes = 0;
                    g->depth = (uint8_t)(sa->depth - (col ? 1 : 0));
                    g->is_store = (uint8_t)sa->store;
                }
            }
        }
    }
    *n_sym = 24 * 2 * 12;
    *n_terms = nt;
    return 0;
}

/* Frames and bind items of the accesses selgen_fill writes for [c0, c1) of
 * config 2 or 5 (in the same order).  values: 9 per nest; items: one per
 * access. */
int selgen_sym_count(int cfg, uint64_t c0, uint64_t c1, uint64_t* n_values, uint64_t* n_items) {
    uint64_t nn = 0, na = 0;
    if ((cfg != SELGEN_C2 && cfg != SELGEN_C5) || selgen_count(cfg, c0, c1, &nn, &na) != 0) return -1;
    *n_values = 9 * nn;
    *n_items = na;
    return 0;
}

int selgen_sym_fill(int cfg, uint64_t c0, uint64_t c1, int64_t* values, gen_bind_item* items) {
    uint64_t nn = 0, na = 0;
    if ((cfg != SELGEN_C2 && cfg != SELGEN_C5) || selgen_count(cfg, c0, c1, &nn, &na) != 0) return -1;
    uint64_t a = 0;
    for (uint64_t i = 0; i < nn; i++) {
        int s, col = 0;
        nest_params np;
        if (cfg == SELGEN_C2) {
            s = c2_nest((int)i, &col);
            shape_params(&SHAPES[s], cfg, 0, col, &np);
        } else {
            uint64_t g = c0 / 32 + i;
            s = (int)(g % 24);
            shape_params(&SHAPES[s], cfg, g / 24, 0, &np);
        }
        int64_t* fr = values + 9 * i;
        fr[FR_ELEM] = np.elem;
        for (int d = 0; d < 4; d++) fr[FR_SIZE + d] = (int64_t)np.symsz[d];
        for (int d = 0; d < 4; d++) fr[FR_OFF + d] = np.arr_off[d];
        for (int k = 0; k < SHAPES[s].n_acc; k++, a++) {
            items[a].sym_access = (uint32_t)((2 * s + col) * 12 + k);
            items[a].frame = (uint32_t)(9 * i);
        }
    }
    return a == na ? 0 : -1;
}
