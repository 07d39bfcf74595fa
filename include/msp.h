/*
 * msp.h -- C ABI of libmsp, the B200 (sm_100a) merge-path sparse library.
 *
 * Implements the data-parallel hot path of S. Dalton, S. Baxter, D. Merrill,
 * L. Olson, M. Garland, "Optimizing Sparse Matrix Operations on GPUs using
 * Merge Path", IPDPS 2015 (PAPER.md, cited as P:<line>):
 *
 *   SpMV    y = A x        merge-path partition + segmented reduction with
 *                          carry-out fix-up (Section III-A)
 *   SpAdd   C = A + B      balanced-path set union of (row,col) tuples in
 *                          two phases, count then fill (III-B)
 *   SpGEMM  C = A B        expand / sort / compress with products balanced
 *                          across CTAs by a search over the prefix sum S of
 *                          the referenced B row lengths (III-C)
 *
 * Every entry point is extern "C", takes plain pointers and sizes, and never
 * exposes a C++ or torch type.  DESIGN.md describes the kernels behind it.
 *
 * Conventions shared by all calls
 * -------------------------------
 * Matrices are CSR: row_offsets int32[nrows+1] with
 * row_offsets[0] == 0 and row_offsets[nrows] == nnz, col_idx int32[nnz],
 * vals float32 or float64 [nnz].  All array pointers in msp_csr and all
 * vector / output / workspace pointers are DEVICE pointers unless the name
 * ends in _host.  SpAdd and SpGEMM require each row's columns to be sorted
 * ascending and unique (the input contract the method relies on);
 * SpMV accepts any column order.  Indices are int32; product counts (Nprods)
 * are int64 internally.
 *
 * Debug validation: with MSP_DEBUG_VALIDATE=1 in the environment (read once
 * per process), msp_spmv, msp_spadd_symbolic and msp_spgemm_setup first run
 * msp_csr_check on their inputs (sorted-unique columns required for SpAdd /
 * SpGEMM), synchronise, and return MSP_ERR_INPUT on a malformed matrix.  The
 * check's flag word lives in the last bytes of the workspace, which is why
 * every *_workspace size includes 512 bytes of tail room.
 *
 * Ownership: the caller allocates and owns every device buffer (inputs,
 * outputs, workspaces).  The library never calls cudaMalloc/cudaFree and
 * keeps no pointer after a call returns, except that the workspaces named in
 * the *_numeric calls must be the ones the matching *_symbolic (or *_setup)
 * call used, left untouched in between.  Workspaces must be zero-filled once
 * before their first use (kernels leave their counters zeroed on exit).
 *
 * Streams: `stream` is a cudaStream_t passed as void* (NULL = legacy default
 * stream).  Calls marked "async" only enqueue work; calls that return a
 * *_host scalar synchronise that stream before returning.
 *
 * Errors: every call returns an msp_status and never aborts.  Argument,
 * shape and dtype checks run on the host before any launch.  Launch errors
 * are returned as MSP_ERR_CUDA with the CUDA error text available from
 * msp_last_error() (thread-local).  Empty inputs are legal (nrows == 0,
 * nnz == 0, all rows empty).  Floating-point results accumulate in fp64
 * and round once to the value type on store (reading Z4); SpAdd
 * values are exact (one IEEE addition per matched pair).  Results are
 * deterministic run to run (no floating-point atomics, fixed carry order).
 */
#ifndef MSP_H_
#define MSP_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define MSP_VERSION 6  /* 2: msp_spgemm_info passed to symbolic / numeric; 3: segmented_rows; 4: msp_set_operation_async, msp_spadd_fused; 5: row_accumulator; 6: small_rows, bitmap_rows */

typedef enum {
    MSP_OK = 0,
    MSP_ERR_ARG = 1,         /* null pointer or negative size */
    MSP_ERR_DTYPE = 2,       /* unsupported or mismatched value type */
    MSP_ERR_SHAPE = 3,       /* A, B, x, y shapes incompatible */
    MSP_ERR_WORKSPACE = 4,   /* workspace too small (query *_workspace) */
    MSP_ERR_OVERFLOW = 5,    /* nnz(C) > INT32_MAX (int32 indices, Z16) */
    MSP_ERR_INPUT = 6,       /* msp_csr_check found a malformed matrix */
    MSP_ERR_CUDA = 7,        /* CUDA launch / runtime error, see msp_last_error */
    MSP_ERR_NCCL = 8,        /* reserved for the multi-GPU layer */
    MSP_ERR_UNSUPPORTED = 9  /* e.g. no sm_100 device */
} msp_status;

typedef enum { MSP_F32 = 0, MSP_F64 = 1 } msp_dtype;

typedef struct {
    int32_t nrows;
    int32_t ncols;
    int64_t nnz;                 /* must equal row_offsets[nrows] */
    const int32_t *row_offsets;  /* device, [nrows+1] */
    const int32_t *col_idx;      /* device, [nnz] */
    const void *vals;            /* device, [nnz] of dtype */
    int32_t dtype;               /* msp_dtype */
} msp_csr;

/* Human-readable name of a status code (static string). */
const char *msp_status_string(int status);
/* Detail of the last error raised on the calling host thread ("" if none). */
const char *msp_last_error(void);
/* MSP_VERSION of the loaded library. */
int msp_version(void);
/* Diagnostics: number of libmsp kernels launched by this process so far
 * (all devices, all threads).  Used by benchmarks to report launches. */
uint64_t msp_launch_count(void);
/* ------------------------------------------------------------------------
 * SpMV  y = A x      (Section III-A)
 *
 * One persistent launch: each CTA takes an equal contiguous range of the
 * merge path of row_end = row_offsets[1..nrows] with the nonzero indices
 * (equal share of rows plus nonzeros), streams its tiles of
 * col_idx/vals through shared memory with TMA bulk copies, gathers x,
 * reduces by row in-tile and emits one (row, partial) carry
 * per CTA; the last CTA to finish adds the carries in CTA order (the update
 * phase; reading Z21).
 *
 * x: device [ncols] of A.dtype.  y: device [nrows] of A.dtype, written
 * entirely (empty rows get +0.0).  ws: device workspace of at least
 * msp_spmv_workspace() bytes, zero-filled before its first use.  Async.
 * ------------------------------------------------------------------------ */
msp_status msp_spmv_workspace(const msp_csr *A, size_t *bytes);
msp_status msp_spmv(const msp_csr *A, const void *x, void *y, void *ws, size_t ws_bytes,
                    void *stream);

/* ------------------------------------------------------------------------
 * SpMV, the paper's own decomposition (ablation):
 * a nonzero-only split -- every CTA gets the same number of nonzeros,
 * Nprods = 2048 -- with the CSR row offsets compacted to the
 * nonempty rows first, a partition kernel (one binary search
 * per CTA segment), a reduction kernel (strided loads, x
 * gathers, strided -> blocked transpose in shared memory, CTA segmented
 * scan) and an update kernel adding every CTA's (row, partial)
 * carry to the row's value (reading Z21).  Same arguments,
 * results and tolerance as msp_spmv (empty rows get +0.0); a row split
 * across CTAs is rounded twice (stored part, then + carries).  Async.
 * ------------------------------------------------------------------------ */
msp_status msp_spmv_nnz_split_workspace(const msp_csr *A, size_t *bytes);
msp_status msp_spmv_nnz_split(const msp_csr *A, const void *x, void *y, void *ws, size_t ws_bytes,
                              void *stream);

/* ------------------------------------------------------------------------
 * SpAdd  C = A + B   (P:496-550 union of (row,col) tuples in Algorithm 1
 * order P:476-490; balanced path P:686-790; two phases P:816-838)
 *
 * A and B: same shape and dtype, sorted unique columns per row.
 * Symbolic: counts the unique tuples of every row of C (cancellations keep
 * an explicit zero, reading Z1), writes C_row_offsets (device int32
 * [nrows+1]) and returns nnz(C) in *nnzC_host; synchronises the stream.
 * Returns MSP_ERR_OVERFLOW if nnz(C) > INT32_MAX.
 * Numeric: fills C_col_idx (device int32 [nnzC]) and C_vals (device
 * [nnzC] of dtype); a matched pair gives (T)(a + b), A's value first
 * (Alg. 1 tie order).  Uses the partition the symbolic call stored in ws.
 * Async.
 * ------------------------------------------------------------------------ */
msp_status msp_spadd_workspace(const msp_csr *A, const msp_csr *B, size_t *bytes);
msp_status msp_spadd_symbolic(const msp_csr *A, const msp_csr *B, int32_t *C_row_offsets,
                              int64_t *nnzC_host, void *ws, size_t ws_bytes, void *stream);
msp_status msp_spadd_numeric(const msp_csr *A, const msp_csr *B, const int32_t *C_row_offsets,
                             int32_t *C_col_idx, void *C_vals, void *ws, size_t ws_bytes,
                             void *stream);

/* One-pass SpAdd (B200 design; same result as symbolic +
 * numeric, bit for bit): the two phases of P:816-838 fused into one tile
 * pass.  Each tile's output offset comes from a decoupled look-back over
 * the tiles' output counts (the tiles' runs of C are contiguous in merge
 * order), and C_row_offsets[r+1] is written at row r's row-end
 * item.  The price is the allocation: C_col_idx / C_vals must hold
 * C_capacity >= nnz(A) + nnz(B) entries (the union's upper bound; else
 * MSP_ERR_SHAPE); C_row_offsets is device int32 [nrows+1].  *nnzC_host
 * receives nnz(C); entries past it are unspecified.  Synchronises the
 * stream.  MSP_ERR_OVERFLOW if nnz(C) > INT32_MAX; MSP_ERR_INPUT if the
 * row-end total and the tile total disagree (unsorted or duplicate
 * columns; stores stay inside C_capacity).  ws: msp_spadd_workspace()
 * bytes. */
msp_status msp_spadd_fused(const msp_csr *A, const msp_csr *B, int32_t *C_row_offsets,
                           int32_t *C_col_idx, void *C_vals, int64_t C_capacity, int64_t *nnzC_host,
                           void *ws, size_t ws_bytes, void *stream);

/* ------------------------------------------------------------------------
 * SpGEMM  C = A B    (ESC: expansion, sorting, compression, P:256-262,
 * P:840-1212, Section III-C)
 *
 * Setup: S = exclusive prefix sum (int64) of the B row lengths
 * referenced by A's column indices, Nprods = S[nnzA], the COO row of every
 * A nonzero, and the classification of rows whose product count exceeds
 * one tile.  Returns the sizes in *info_host; synchronises the stream once.
 * Symbolic: products are partitioned into tiles by a merge-path search over
 * (S, product index) (reading Z7), expanded, sorted by
 * (row, col) with a block merge sort and compressed; rows that straddle a
 * tile boundary and rows longer than a tile are completed by a second pass
 * (the paper's global phase).  Writes C_row_offsets and
 * *nnzC_host and records the largest tile row span in info_host (in/out:
 * pass the struct setup filled); synchronises the stream twice (the tile
 * key width depends on that span; nnz(C)).  MSP_ERR_OVERFLOW if nnz(C) >
 * INT32_MAX.  The symbolic pass keeps every tile's sorting permutation in
 * main_ws (2 bytes per tile slot, as the paper stores the CTA sort's
 * permutation).
 * Numeric: re-expands the products with values, applies the stored
 * permutation (no second sort) and compresses; the long-row pass is repeated
 * with values.  Writes C_col_idx / C_vals; fp64 accumulation in a fixed,
 * deterministic order.  Must follow msp_spgemm_symbolic on the same
 * setup_ws / main_ws, with A and B unchanged, and get the info_host that
 * symbolic updated (MSP_ERR_ARG if max_tile_span is unset).  Async: no
 * synchronisation, every size comes from info_host.
 * setup_ws: msp_spgemm_setup_workspace() bytes; main_ws: info.main_ws_bytes.
 * ------------------------------------------------------------------------ */
typedef struct {
    int64_t nprods;          /* sum over A nonzeros of nnz(B row col) */
    int64_t ntiles;          /* product tiles of the main pass */
    int64_t long_rows;       /* rows with more products than one tile */
    int64_t long_products;   /* products in those rows */
    int64_t max_row_products;
    int64_t main_ws_bytes;   /* size of the main workspace */
    int64_t long_chunks;     /* sorted chunks of the long-row pass */
    int64_t max_tile_span;   /* largest row span of a product tile: -1 after
                                setup, set by symbolic (picks the key width) */
    int64_t segmented_rows;  /* windows (CTAs) of the long rows taking the
                                segmented (dense accumulator) path instead of
                                the ESC long-row pass: >= 1 product per 4
                                columns of the output span; a span wider than
                                12,288 columns is cut into 12,288-column
                                windows while windows x nnz(A row) <=
                                products (one window per row otherwise, so
                                for narrow rows this counts rows; SURVEY §8(f)
                                f3; MSP_SPGEMM_SEGMENTED=0 disables) */
    int64_t row_accumulator; /* > 0: every short row's output span is at most
                                65,536 columns (the value is the widest
                                span, which sizes the bitmaps), so the short
                                rows take the
                                row-accumulator path (a warp per row: bitmap
                                count in symbolic, shared-memory accumulation
                                in k order in numeric) and no product tile
                                runs; 0: the ESC tile pass.  main_ws then holds
                                one int32 per product (each short row's column
                                list) instead of the tile permutations.
                                MSP_SPGEMM_ROWACC=0 disables (ablation). */
    int64_t small_rows;      /* short rows with at most 64 products taking the
                                compare-count path (a warp per batch of
                                consecutive rows with <= 256 products: each
                                product's rank from the first occurrences of
                                its row, k-ordered sums; no column list in
                                main_ws).  Short rows with more products whose
                                span exceeds 65,536 columns are promoted to
                                long rows, so the warp-row path covers every
                                short row.  MSP_SPGEMM_SMALL=0 disables (the
                                v5 behaviour: one too-wide row sends every
                                short row to the ESC tiles). */
    int64_t bitmap_rows;     /* short rows taking the bitmap / hash path */
} msp_spgemm_info;

msp_status msp_spgemm_setup_workspace(const msp_csr *A, const msp_csr *B, size_t *bytes);
msp_status msp_spgemm_setup(const msp_csr *A, const msp_csr *B, void *setup_ws,
                            size_t setup_ws_bytes, msp_spgemm_info *info_host, void *stream);
msp_status msp_spgemm_symbolic(const msp_csr *A, const msp_csr *B, const void *setup_ws,
                               size_t setup_ws_bytes, void *main_ws, size_t main_ws_bytes,
                               msp_spgemm_info *info_host, int32_t *C_row_offsets,
                               int64_t *nnzC_host, void *stream);
msp_status msp_spgemm_numeric(const msp_csr *A, const msp_csr *B, const void *setup_ws,
                              size_t setup_ws_bytes, void *main_ws, size_t main_ws_bytes,
                              const msp_spgemm_info *info_host, const int32_t *C_row_offsets,
                              int32_t *C_col_idx, void *C_vals, void *stream);

/* ------------------------------------------------------------------------
 * SpGEMM with the paper's own sort pipeline (ablation, SURVEY §8(f) f2;
 * P:994-1212, Figs 3-4).  After msp_spgemm_setup (same setup_ws / info):
 * symbolic = phase 1 (per tile of 2048 products: expand (row, col), one
 * keys-only radix sort on the ceil(log2 n) column bits with the tile index
 * in the low bits, duplicates adjacent, 16-bit permutation + head flags
 * stored, reduced entries compacted in tile order) and phase 2 (a global
 * LSD radix sort of the reduced (row, col) keys that only computes their
 * permutation), then C.row_offsets and *nnz_C (synchronises twice).
 * Numeric = phase 3 (re-expansion with values, each tile's stored
 * permutation, reduction by the stored duplicate flags, values stored at
 * their sorted positions) and a global reduce-by-key into C (async).  Same
 * results as msp_spgemm_* (structure bit-exact, values within tolerance,
 * deterministic); Nprods must be < 2^32.  ws: msp_spgemm_radix_workspace()
 * bytes, untouched between symbolic and numeric.
 * ------------------------------------------------------------------------ */
msp_status msp_spgemm_radix_workspace(const msp_csr *A, const msp_csr *B, const msp_spgemm_info *info_host,
                                      size_t *bytes);
msp_status msp_spgemm_radix_symbolic(const msp_csr *A, const msp_csr *B, const void *setup_ws,
                                     size_t setup_ws_bytes, void *ws, size_t ws_bytes,
                                     const msp_spgemm_info *info_host, int32_t *C_row_offsets,
                                     int64_t *nnzC_host, void *stream);
msp_status msp_spgemm_radix_numeric(const msp_csr *A, const msp_csr *B, const void *setup_ws,
                                    size_t setup_ws_bytes, void *ws, size_t ws_bytes,
                                    const msp_spgemm_info *info_host, const int32_t *C_row_offsets,
                                    int32_t *C_col_idx, void *C_vals, void *stream);

/* ------------------------------------------------------------------------
 * Input validation (the CSR contract of P:316-322).
 * flags_host receives a bit set: 1 = row_offsets not monotone or
 * row_offsets[0] != 0 or row_offsets[nrows] != nnz, 2 = column out of
 * [0, ncols), 4 = columns not strictly increasing within a row (only
 * checked when require_sorted_unique != 0).  Returns MSP_ERR_INPUT if any
 * flag is set.  ws: at least 16 bytes, zero-filled.  Synchronises.
 * ------------------------------------------------------------------------ */
msp_status msp_csr_check(const msp_csr *A, int require_sorted_unique, int32_t *flags_host,
                         void *ws, size_t ws_bytes, void *stream);

/* ------------------------------------------------------------------------
 * Set operations on sorted key lists (the paper's second
 * contribution, Fig 2).  A_keys[nA], B_keys[nB]: device,
 * sorted ascending as unsigned integers of key_bytes (4 or 8) bytes;
 * duplicates allowed.  A_vals / B_vals: device payloads of val_bytes (0, 4 or
 * 8; NULL when 0) per key, carried bit-for-bit.  Duplicates are key-rank
 * pairs: the r-th copy of a key in A matches the r-th copy in B (P:700-712,
 * reading R4), so with cA / cB copies of a key the result holds
 *   MSP_SET_UNION                 max(cA, cB) copies (matched from A),
 *   MSP_SET_INTERSECTION          min(cA, cB) copies (from A),
 *   MSP_SET_DIFFERENCE            max(cA - cB, 0) copies (A - B),
 *   MSP_SET_SYMMETRIC_DIFFERENCE  |cA - cB| copies (longer side),
 * ascending.  C_keys / C_vals: device, capacity C_capacity entries, which
 * must be at least nA + nB (union, symmetric difference), min(nA, nB)
 * (intersection) or nA (difference), else MSP_ERR_SHAPE.  *nC_host receives
 * the result size.  ws: msp_set_op_workspace() bytes, caller-owned.
 * Synchronises the stream (returns the size).  Keys not sorted ascending
 * (as unsigned integers; a signed tensor holding negatives is not) give
 * MSP_ERR_INPUT: every tile checks its windows while staging them, reads
 * and writes stay inside the given arrays and C_capacity, and the contents
 * of C are then unspecified.
 * ------------------------------------------------------------------------ */
typedef enum {
    MSP_SET_UNION = 0,
    MSP_SET_INTERSECTION = 1,
    MSP_SET_DIFFERENCE = 2,
    MSP_SET_SYMMETRIC_DIFFERENCE = 3
} msp_set_op;

msp_status msp_set_op_workspace(int64_t nA, int64_t nB, size_t *bytes);
msp_status msp_set_operation(msp_set_op op, const void *A_keys, const void *A_vals, int64_t nA,
                             const void *B_keys, const void *B_vals, int64_t nB, int32_t key_bytes,
                             int32_t val_bytes, void *C_keys, void *C_vals, int64_t C_capacity,
                             int64_t *nC_host, void *ws, size_t ws_bytes, void *stream);

/* The same operation without the host round trip: nC_dev is a DEVICE
 * int64[2] (8-byte aligned, caller-owned) that receives, in stream order,
 * nC_dev[0] = the result size and nC_dev[1] != 0 iff the keys were found
 * unsorted (the MSP_ERR_INPUT condition of msp_set_operation, which this
 * call cannot return).  Async: two launches (partition, which also clears
 * the look-back state, and the tile kernel), no stream synchronisation, no
 * device-to-host copy -- for pipelines that consume the result on the GPU
 * (e.g. a size-bounded next step reading nC_dev) and for the Fig 2 rate
 * without the per-call host sync.  ws must stay reserved until the stream
 * reaches the end of the call. */
msp_status msp_set_operation_async(msp_set_op op, const void *A_keys, const void *A_vals, int64_t nA,
                                   const void *B_keys, const void *B_vals, int64_t nB, int32_t key_bytes,
                                   int32_t val_bytes, void *C_keys, void *C_vals, int64_t C_capacity,
                                   int64_t *nC_dev, void *ws, size_t ws_bytes, void *stream);

/* ------------------------------------------------------------------------
 * Multi-GPU helpers.  Row blocks are balanced by nnz:
 * rank r owns rows [R_r, R_{r+1}), R_r = lower_bound(row_offsets,
 * ceil(r * nnz / P)), R_0 = 0, R_P = nrows.  row_offsets_host is a HOST
 * array [nrows+1]; row_starts_host a HOST array [P+1].  Pure host code.
 * ------------------------------------------------------------------------ */
msp_status msp_row_split(const int32_t *row_offsets_host, int32_t nrows, int32_t P,
                         int32_t *row_starts_host);

/* Rebase a row-offset array on the device: out[i] = in[i] - in[0] + base,
 * i in [0, n); `in` and `out` must not alias.  Used to form row-block views
 * and to concatenate gathered blocks.  Async. */
msp_status msp_rebase_offsets(const int32_t *in, int32_t *out, int64_t n, int64_t base,
                              void *stream);

/* Gather dst[i] = src[idx[i]], i in [0, n), of value_bytes (4 or 8) each:
 * packs the halo values a rank sends to its neighbours in the distributed
 * SpMV without full-x replication.
 * Device pointers; idx entries must be valid indices of src.  Async. */
msp_status msp_gather_values(const void *src, const int32_t *idx, int64_t n, int32_t value_bytes, void *dst,
                             void *stream);

#ifdef __cplusplus
}
#endif
#endif /* MSP_H_ */
