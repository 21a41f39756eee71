/*
 * rap_oracle.h — CPU ORACLE for RAP's DLRM input-preprocessing operators.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference legs may load this library.
 * The product path (include/rap.h, paper_conf_asplos_wangwdz0d24_b200/) never
 * includes, links or calls anything here, and this file includes nothing from
 * the product path.  The two implementations share no code.
 *
 * What it computes: the plain, row-by-row definition of every operator of
 * PAPER.md Table 1 (L440-463) under the readings listed in DESIGN.md §3.
 * RAP's fusion, sharding, scheduling and mapping change WHERE and WHEN
 * operators run, never WHAT they compute (§6.1,
 * L1351-1366 §6.2, L1526-1534 §7.2), so the oracle evaluates each output's
 * DAG (L718-720 §2.3) on each row independently, one op at a time.
 *
 * Parity status per function: see the header of rap_oracle.c and DESIGN.md §4.
 */
#ifndef RAP_ORACLE_H
#define RAP_ORACLE_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* Status codes (same numeric meaning as the product's, compared by name in tests). */
enum {
  ORC_OK = 0,
  ORC_ERR_INVALID_ARGUMENT = 1,
  ORC_ERR_INVALID_GRAPH = 2,
  ORC_ERR_INVALID_PARAM = 3,
  ORC_ERR_CAPACITY = 4,
  ORC_ERR_UNSUPPORTED = 5,
  ORC_ERR_NOMEM = 7
};

/* Operators, Table 1 (L440-463). */
enum {
  ORC_FILLNULL = 0,   /* L462 */
  ORC_LOGIT = 1,      /* L446 */
  ORC_BOXCOX = 2,     /* L448 */
  ORC_ONEHOT = 3,     /* L449 */
  ORC_SIGRIDHASH = 4, /* L452 */
  ORC_BUCKETIZE = 5,  /* L458 */
  ORC_FIRSTX = 6,     /* L454 */
  ORC_CLAMP = 7,      /* L455 */
  ORC_NGRAM = 8,      /* L459, footnote L181-182 */
  ORC_MAPID = 9       /* L460 */
};

/* Where a node input comes from. */
enum { ORC_IN_NODE = 0, ORC_IN_DENSE = 1, ORC_IN_SPARSE = 2 };

#define ORC_MAX_IN 8

typedef struct {
  int32_t op;
  int32_t n_in;
  int32_t in_kind[ORC_MAX_IN];
  int32_t in_idx[ORC_MAX_IN];
  /* parameters (only the ones the op uses are read) */
  float f_fill;      /* FillNull on a dense value */
  float eps;         /* Logit */
  float lambda;      /* BoxCox */
  int64_t i_fill;    /* FillNull on an id list */
  int64_t lo, hi;    /* Clamp */
  int64_t x;         /* FirstX */
  int64_t max_value; /* SigridHash / NGram table size M */
  int64_t map_default;
  uint64_t salt;     /* SigridHash / NGram */
  int32_t n;         /* NGram window */
  int32_t k_width;   /* OneHot K */
  int32_t n_borders; /* Bucketize m */
  const float* f_borders;   /* Bucketize of a dense value */
  const int64_t* i_borders; /* Bucketize of an id list */
  int64_t map_size;
  const int64_t* map_keys;
  const int64_t* map_vals;
} orc_node;

typedef struct {
  int32_t n_dense, n_sparse, n_nodes;
  const orc_node* nodes;
  int32_t n_outputs;
  const int32_t* outputs; /* node indices, in output order */
} orc_graph;

/* Host arrays.  Validity bitmaps: bit (b & 31) of word (b >> 5), 1 = valid;
 * a NULL bitmap means every row is valid.  Offsets are absolute (Arrow). */
typedef struct {
  int64_t n_rows;
  const float* const* dense;
  const uint32_t* const* dense_valid;
  const int32_t* const* sp_off;
  const int64_t* const* sp_val;
  const uint32_t* const* sp_valid;
} orc_batch;

/* Outputs, allocated by orc_run, released by orc_free. */
typedef struct {
  int64_t n_rows, d_out, f_out, n_values;
  float* dense;     /* [n_rows x d_out] row-major */
  int32_t* lengths; /* [f_out x n_rows] feature-major */
  int64_t* offsets; /* [f_out x n_rows + 1] */
  int64_t* values;  /* [n_values] (feature, row, element) order */
} orc_result;

int orc_validate(const orc_graph* g, int64_t* d_out, int64_t* f_out);
int orc_run(const orc_graph* g, const orc_batch* b, orc_result* r);
void orc_free(orc_result* r);

/* Scalar entry points used by the pin tests. */
uint64_t orc_H(uint64_t x);
uint64_t orc_reduce(uint64_t h, int64_t M);
int64_t orc_sigridhash(int64_t x, uint64_t salt, int64_t M);
float orc_logit(float x, float eps);
float orc_boxcox(float x, float lambda);
int64_t orc_bucketize_f(float x, const float* borders, int32_t m);
int64_t orc_bucketize_i(int64_t x, const int64_t* borders, int32_t m);
int64_t orc_ngram(const int64_t* c, int64_t len, int32_t n, uint64_t salt, int64_t M, int64_t* out);

#ifdef __cplusplus
}
#endif
#endif
