/*
 * ds_oracle.c -- CPU ORACLE for the in-place Data Sliding primitives.
 *
 * TEST INFRASTRUCTURE ONLY (see ds_oracle.h): only tests/, smoke() and
 * bench.py's cpu_baseline / --impl reference legs may use it.
 *
 * Each function is the plain sequential definition from PAPER.md, in place,
 * reading every element before anything can overwrite it because the write
 * index never passes the read index (compaction-like ops) or because rows
 * are moved in the order the paper prescribes (pad: last row first).
 * No blocking, tiling, fusion or parallelism.
 */
#include "ds_oracle.h"

#include <string.h>

/* Reinterpret the 32-bit pattern as int32 / float without aliasing UB. */
static int32_t as_i32(uint32_t w) { int32_t x; memcpy(&x, &w, 4); return x; }
static float as_f32(uint32_t w) { float x; memcpy(&x, &w, 4); return x; }

/* Predicates of the select primitive (Fig. 11 uses "element value
 * is even").  Ids are fixed by the ds_select ABI.                */
int oracle_predicate(int pred, uint32_t w, uint32_t param) {
    switch (pred) {
    case ORACLE_PRED_NONZERO:    return w != 0u;
    case ORACLE_PRED_I32_GT:     return as_i32(w) > as_i32(param);
    case ORACLE_PRED_I32_NOT_GT: return !(as_i32(w) > as_i32(param));
    case ORACLE_PRED_F32_GT:     return as_f32(w) > as_f32(param);
    case ORACLE_PRED_F32_NOT_GT: return !(as_f32(w) > as_f32(param));
    case ORACLE_PRED_I32_EVEN:   return (as_i32(w) % 2) == 0;
    case ORACLE_PRED_I32_ODD:    return (as_i32(w) % 2) != 0;
    default:                     return -1;
    }
}

/* P:244 stream compaction: drop words equal to remove_value, keep order.
 * Write index w <= read index i, so a[i] is still the original when read. */
size_t oracle_compact(uint32_t* a, size_t n, uint32_t remove_value) {
    size_t w = 0;
    for (size_t i = 0; i < n; ++i) {
        uint32_t x = a[i];
        if (x != remove_value) a[w++] = x;
    }
    return w;
}

/* P:232 select: keep words for which the predicate is true, keep order. */
size_t oracle_select(uint32_t* a, size_t n, int pred, uint32_t param) {
    if (pred < 0 || pred >= ORACLE_PRED_COUNT) return (size_t)-1;
    size_t w = 0;
    for (size_t i = 0; i < n; ++i) {
        uint32_t x = a[i];
        if (oracle_predicate(pred, x, param)) a[w++] = x;
    }
    return w;
}

/* P:264 unique with an optional predecessor word for element 0.
 * `prev` always holds the ORIGINAL a[i-1]: it is copied before a[w] may
 * overwrite anything, and w <= i.                                        */
size_t oracle_unique_prev(uint32_t* a, size_t n, int has_prev, uint32_t prev) {
    size_t w = 0;
    for (size_t i = 0; i < n; ++i) {
        uint32_t cur = a[i];
        int keep = (i == 0) ? (!has_prev || cur != prev) : (cur != prev);
        if (keep) a[w++] = cur;
        prev = cur;
    }
    return w;
}

size_t oracle_unique(uint32_t* a, size_t n) {
    return oracle_unique_prev(a, n, 0, 0u);
}

/* P:286-292 partition: true words first, then false words, both in input
 * order.  The false words go to aux (the paper's Array_false) and are
 * copied back to the tail "once the true elements have been shifted".     */
size_t oracle_partition(uint32_t* a, size_t n, int pred, uint32_t param, uint32_t* aux) {
    if (pred < 0 || pred >= ORACLE_PRED_COUNT) return (size_t)-1;
    size_t t = 0, f = 0;
    for (size_t i = 0; i < n; ++i) {
        uint32_t x = a[i];
        if (oracle_predicate(pred, x, param)) a[t++] = x;
        else aux[f++] = x;
    }
    for (size_t j = 0; j < f; ++j) a[t + j] = aux[j];
    return t;
}

/* P:242 DS Copy_if: out-of-place select. */
size_t oracle_select_copy(const uint32_t* in, size_t n, int pred, uint32_t param,
                          uint32_t* out) {
    if (pred < 0 || pred >= ORACLE_PRED_COUNT) return (size_t)-1;
    size_t w = 0;
    for (size_t i = 0; i < n; ++i)
        if (oracle_predicate(pred, in[i], param)) out[w++] = in[i];
    return w;
}

/* "move each row starting from the last one"; row r goes from byte
 * offset r*cols*eb to r*new_cols*eb (a shift of (new_cols-cols)*r elements,
 * "row i will be shifted by C x i"), then its new cells get the fill.    */
int oracle_pad(uint8_t* b, size_t rows, size_t cols, size_t new_cols,
               size_t elem_bytes, const uint8_t* fill) {
    if (new_cols < cols || elem_bytes == 0) return -1;
    for (size_t r = rows; r-- > 0;) {
        uint8_t* dst = b + r * new_cols * elem_bytes;
        const uint8_t* src = b + r * cols * elem_bytes;
        memmove(dst, src, cols * elem_bytes);
        for (size_t c = cols; c < new_cols; ++c) {
            uint8_t* cell = dst + c * elem_bytes;
            if (fill) memcpy(cell, fill, elem_bytes);
            else memset(cell, 0, elem_bytes);
        }
    }
    return 0;
}

/* unpadding "removes the extra columns": keep the first new_cols
 * elements of each row; rows move backwards, so go from the first row on. */
int oracle_unpad(uint8_t* b, size_t rows, size_t cols, size_t new_cols,
                 size_t elem_bytes) {
    if (new_cols > cols || elem_bytes == 0) return -1;
    for (size_t r = 0; r < rows; ++r) {
        memmove(b + r * new_cols * elem_bytes, b + r * cols * elem_bytes,
                new_cols * elem_bytes);
    }
    return 0;
}

/* every element of the single group moves by the same constant; the
 * move is backward, so go from the first element on (no element is
 * overwritten before it was moved).                                      */
int oracle_slide(uint8_t* b, size_t n, size_t shift, size_t elem_bytes) {
    if (shift > n || elem_bytes == 0) return -1;
    for (size_t i = shift; i < n; ++i)
        for (size_t k = 0; k < elem_bytes; ++k)
            b[(i - shift) * elem_bytes + k] = b[i * elem_bytes + k];
    return 0;
}

/* 8-byte elements: the same sequential definitions on 64-bit patterns. */
int oracle_predicate64(int pred, uint64_t e, uint64_t param) {
    double de, dp;
    memcpy(&de, &e, sizeof de);
    memcpy(&dp, &param, sizeof dp);
    switch (pred) {
    case ORACLE_PRED_NONZERO: return e != 0;
    case ORACLE_PRED_I32_GT: return (int64_t)e > (int64_t)param;
    case ORACLE_PRED_I32_NOT_GT: return !((int64_t)e > (int64_t)param);
    case ORACLE_PRED_F32_GT: return de > dp;
    case ORACLE_PRED_F32_NOT_GT: return !(de > dp);
    case ORACLE_PRED_I32_EVEN: return (e & 1u) == 0;
    case ORACLE_PRED_I32_ODD: return (e & 1u) != 0;
    default: return -1;
    }
}

size_t oracle_compact64(uint64_t* a, size_t n, uint64_t remove_value) {
    size_t w = 0;
    for (size_t i = 0; i < n; ++i)
        if (a[i] != remove_value) a[w++] = a[i];
    return w;
}

size_t oracle_select64(uint64_t* a, size_t n, int pred, uint64_t param) {
    if (pred < 0 || pred >= ORACLE_PRED_COUNT) return (size_t)-1;
    size_t w = 0;
    for (size_t i = 0; i < n; ++i)
        if (oracle_predicate64(pred, a[i], param)) a[w++] = a[i];
    return w;
}

size_t oracle_unique64(uint64_t* a, size_t n) {
    if (n == 0) return 0;
    uint64_t prev = a[0];
    size_t w = 1;
    for (size_t i = 1; i < n; ++i) {
        const uint64_t cur = a[i];
        if (cur != prev) a[w++] = cur;
        prev = cur;
    }
    return w;
}
