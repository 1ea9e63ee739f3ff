/*
 * ds_oracle.h -- CPU ORACLE for the in-place Data Sliding (DS) primitives.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and the
 * cpu_baseline / --impl reference legs of bench.py may load, call, link or
 * execute anything under oracle/.  The product path (libds) never does; it
 * shares no code, header, table or constant generator with this file.
 *
 * Plain, sequential, single-threaded C.  Every function is the textbook
 * definition of its primitive, written out in the paper's terms:
 *   PAPER.md = /root/reference/PAPER.md (Gomez-Luna et al., ICPP 2015);
 *   "P:NN" = line NN of that file.
 *
 * Element type: the paper's arrays are 4-byte int/float (P:242, P:248,
 * "single precision"); compact/select/unique therefore work on
 * 32-bit words.  Pad/unpad work on rows of elem_bytes-sized elements
 * (float and double).
 *
 * Equality is BITWISE on the 32-bit pattern (reading R13).
 *
 * Parity status: every function here is pinned by tests/test_oracle_pins.py
 * (brute force, C++ std:: library routines, numpy.pad, closed forms,
 * invariants, golden fixtures).  None is "parity unpinned".
 */
#ifndef DS_ORACLE_H
#define DS_ORACLE_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* Predicate ids: the numeric values are the documented ABI of ds_select
 * (include/ds.h); they are re-declared here, NOT included, so the oracle
 * shares no header with the product.                                      */
enum {
    ORACLE_PRED_NONZERO    = 0, /* w != 0 (bitwise)                          */
    ORACLE_PRED_I32_GT     = 1, /* (int32)w >  (int32)param                 */
    ORACLE_PRED_I32_NOT_GT = 2, /* !((int32)w > (int32)param)               */
    ORACLE_PRED_F32_GT     = 3, /* (float)w >  (float)param, NaN -> false   */
    ORACLE_PRED_F32_NOT_GT = 4, /* !((float)w > (float)param)               */
    ORACLE_PRED_I32_EVEN   = 5, /* (int32)w is even       (Fig. 11)  */
    ORACLE_PRED_I32_ODD    = 6, /* (int32)w is odd                          */
    ORACLE_PRED_COUNT      = 7
};

/* Evaluate predicate `pred` on word w with parameter bits `param`.
 * Returns 1 (true), 0 (false) or -1 (unknown predicate id).             */
int oracle_predicate(int pred, uint32_t w, uint32_t param);

/* Stream compaction: "eliminates those elements of the array that
 * are equal to a certain value".  Stable, in place.  Returns the
 * number of kept words; a[0..ret) holds them in input order; a[ret..n) is
 * left as it was (reading R5).                                           */
size_t oracle_compact(uint32_t* a, size_t n, uint32_t remove_value);

/* Select: "filters elements according to the evaluation of a
 * certain predicate"; this version KEEPS predicate-true words (reading
 * R14).  Returns (size_t)-1 for an unknown predicate id (a untouched).    */
size_t oracle_select(uint32_t* a, size_t n, int pred, uint32_t param);

/* Unique: "For each group of consecutive elements that are equal in
 * the input array, it removes all but the first of these".  Word i is kept
 * iff i == 0 or a[i] != a[i-1] (original values).                        */
size_t oracle_unique(uint32_t* a, size_t n);

/* Unique of one shard of a longer array (multi-GPU, R18):
 * word 0 is compared with `prev` when has_prev != 0, else it is kept.    */
size_t oracle_unique_prev(uint32_t* a, size_t n, int has_prev, uint32_t prev);

/* Partition: "The elements that satisfy the predicate are
 * placed in the first part of the array, preceding the elements that do not
 * satisfy the predicate"; stable for both classes (the DS stability of P:15;
 * the paper compares with thrust::stable_partition).  In place on a;
 * `aux` (n words) plays the paper's auxiliary Array_false.  Returns the
 * number of true words, or (size_t)-1 for an unknown predicate.           */
size_t oracle_partition(uint32_t* a, size_t n, int pred, uint32_t param, uint32_t* aux);

/* Out-of-place select ("DS Copy_if"): the predicate-true words
 * of in[0, n) are written in order to out; in is not modified.           */
size_t oracle_select_copy(const uint32_t* in, size_t n, int pred, uint32_t param,
                          uint32_t* out);

/* Padding: rows x cols matrix (row-major, elem_bytes per element)
 * at b; the buffer has room for rows x new_cols elements ("the extra memory
 * space needs to be previously allocated adjacent to the matrix").
 * Row i moves forward by (new_cols-cols)*i elements; rows are moved
 * "starting from the last one" ([13]); the new trailing cells of each
 * row receive `fill` (elem_bytes bytes; NULL = zero bytes; reading R2).
 * Returns 0, or -1 if new_cols < cols or elem_bytes == 0.                */
int oracle_pad(uint8_t* b, size_t rows, size_t cols, size_t new_cols,
               size_t elem_bytes, const uint8_t* fill);

/* Unpadding: "removes the extra columns" -- keeps the first
 * new_cols elements of every row, rows moved from the first one on.
 * Bytes past rows*new_cols*elem_bytes are left as they were (R5).
 * Returns 0, or -1 if new_cols > cols or elem_bytes == 0.                */
int oracle_unpad(uint8_t* b, size_t rows, size_t cols, size_t new_cols,
                 size_t elem_bytes);

/* 8-byte elements (int64 / float64 bit patterns).  Same
 * definitions as the 32-bit functions above with 64-bit elements: compaction
 * removes elements bitwise-equal to the value; select keeps predicate-true
 * elements, the predicate ids widened (I32 -> int64, F32 -> double, EVEN/ODD
 * on bit 0); unique keeps element i iff i == 0 or a[i] != a[i-1].         */
int oracle_predicate64(int pred, uint64_t e, uint64_t param);
size_t oracle_compact64(uint64_t* a, size_t n, uint64_t remove_value);
size_t oracle_select64(uint64_t* a, size_t n, int pred, uint64_t param);
size_t oracle_unique64(uint64_t* a, size_t n);

/* Slide, the one-group regular DS ("groups of consecutive input
 * array elements are shifted by a constant amount of memory positions"):
 * elements [shift, n) (elem_bytes each) move backward by `shift` to
 * [0, n - shift), in input order; elements [n - shift, n) keep their bytes
 * (R5).  Returns 0, or -1 if shift > n or elem_bytes == 0.               */
int oracle_slide(uint8_t* b, size_t n, size_t shift, size_t elem_bytes);

#ifdef __cplusplus
}
#endif
#endif /* DS_ORACLE_H */
