/*
 * cswap_oracle.c — plain, slow, obviously-correct CPU oracle for the CSWAP hot path.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load this library.  The product path
 * (paper_conf_cluster_chenhzchysc21_b200/) never links, imports or executes it, and it
 * shares no code, header or constant table with csrc/.
 *
 * Paper: "CSWAP: A Self-Tuning Compression Framework for Accelerating Tensor Swapping
 * in GPUs" (Chen et al., CLUSTER'21), cited as PAPER.md:<line> (§, Eq.).
 * Byte format: DESIGN.md §3 "Canonical container v1" (the paper is silent on bytes;
 * every reading is listed in DESIGN.md §2).
 *
 * Style rules: scalar loops in the paper's order, no blocking, no SIMD, no tricks.
 * Elements are raw w-byte words (w = 4 for f32, 2 for f16/bf16) compared BITWISE.
 *
 * Parity status: every function below is pinned by tests/test_oracle_*.py against
 * something other than itself (paper worked examples, closed forms, numpy/scipy,
 * liblz4 1.9.4, brute force).  No function is "parity unpinned".
 */
#include <stdint.h>
#include <stddef.h>
#include <string.h>
#include <math.h>
#include <stdlib.h>

#define ORC_OK 0
#define ORC_ERR_INVALID (-1)
#define ORC_ERR_CAPACITY (-4)
#define ORC_ERR_CORRUPT (-5)

enum { C_NONE = 0, C_ZVC = 1, C_RLE = 2, C_CSR = 3, C_LZ4 = 4 };
enum { D_F32 = 0, D_F16 = 1, D_BF16 = 2 };

/* ------------------------------------------------------------------------- */
/* little helpers                                                             */
/* ------------------------------------------------------------------------- */
static uint64_t align16(uint64_t x) { return (x + 15) / 16 * 16; }
static uint64_t ceil_div(uint64_t a, uint64_t b) { return (a + b - 1) / b; }

static int width_of(int dtype) {
    if (dtype == D_F32) return 4;
    if (dtype == D_F16 || dtype == D_BF16) return 2;
    return 0;
}

/* element i as an unsigned word (bitwise view; reading "zero" = all bits 0, R1) */
static uint32_t elem(const uint8_t* p, uint64_t i, int w) {
    uint32_t v = 0;
    for (int b = 0; b < w; b++) v |= (uint32_t)p[i * w + b] << (8 * b);
    return v;
}
static void put_elem(uint8_t* p, uint64_t i, int w, uint32_t v) {
    for (int b = 0; b < w; b++) p[i * w + b] = (uint8_t)(v >> (8 * b));
}
static void put_u16(uint8_t* p, uint16_t v) { p[0] = (uint8_t)v; p[1] = (uint8_t)(v >> 8); }
static void put_u32(uint8_t* p, uint32_t v) { for (int b = 0; b < 4; b++) p[b] = (uint8_t)(v >> (8 * b)); }
static void put_u64(uint8_t* p, uint64_t v) { for (int b = 0; b < 8; b++) p[b] = (uint8_t)(v >> (8 * b)); }
static uint32_t get_u16(const uint8_t* p) { return (uint32_t)p[0] | ((uint32_t)p[1] << 8); }
static uint32_t get_u32(const uint8_t* p) {
    return (uint32_t)p[0] | ((uint32_t)p[1] << 8) | ((uint32_t)p[2] << 16) | ((uint32_t)p[3] << 24);
}
static uint64_t get_u64(const uint8_t* p) {
    uint64_t v = 0;
    for (int b = 0; b < 8; b++) v |= (uint64_t)p[b] << (8 * b);
    return v;
}

/* ------------------------------------------------------------------------- */
/* Container v1 geometry                                       */
/* ------------------------------------------------------------------------- */
static uint64_t data_start(uint32_t K) { return align16(64 + 8 * (uint64_t)K); }
static uint64_t frame_elems(uint64_t n, uint64_t F, uint64_t k) {
    uint64_t s = k * F, e = s + F;
    if (e > n) e = n;
    return e - s;
}

/* ------------------------------------------------------------------------- */
/* Frame payload encoders.  Each writes exactly the payload bytes (sections   */
/* zero-padded to 16) into `out` (which the caller zeroed) and returns the    */
/* frame byte count.                                                          */
/* ------------------------------------------------------------------------- */

/* NONE: raw bytes.  (vDNN-style uncompressed swap) */
static uint64_t enc_none(const uint8_t* x, uint64_t Fk, int w, uint8_t* out) {
    memcpy(out, x, Fk * (uint64_t)w);
    return align16(Fk * (uint64_t)w);
}

/* ZVC — PAPER.md:222 (§IV-E): "it utilizes a 32-bit bitmap as the index for 32
 * consecutive floats" + the non-zero values.  Bit j of word i <-> element 32i+j,
 * 1 = non-zero (R2).                                                */
static uint64_t enc_zvc(const uint8_t* x, uint64_t Fk, int w, uint8_t* out) {
    uint64_t nwords = ceil_div(Fk, 32);
    uint64_t bm_bytes = align16(4 * nwords);
    for (uint64_t i = 0; i < nwords; i++) {
        uint32_t word = 0;
        for (uint64_t j = 0; j < 32; j++) {
            uint64_t e = 32 * i + j;
            if (e < Fk && elem(x, e, w) != 0) word |= (uint32_t)1 << j;
        }
        put_u32(out + 4 * i, word);
    }
    uint64_t nnz = 0;
    for (uint64_t e = 0; e < Fk; e++) {
        uint32_t v = elem(x, e, w);
        if (v != 0) {
            put_elem(out + bm_bytes, nnz, w, v);
            nnz++;
        }
    }
    return bm_bytes + align16(nnz * (uint64_t)w);
}

/* RLE — PAPER.md:220 (§IV-E): "stores data sequences where the same value occurs in
 * many consecutive positions as a single value and count".  Every maximal run of
 * bitwise-equal words becomes (length, value); no run-of-1 elision (R4).
 * Frame: {u32 r, 12 zero bytes} | u32 lengths[r] pad16 | values[r] pad16.         */
static uint64_t enc_rle(const uint8_t* x, uint64_t Fk, int w, uint8_t* out) {
    /* pass 1: count runs */
    uint64_t r = 0;
    for (uint64_t e = 0; e < Fk; e++)
        if (e == 0 || elem(x, e, w) != elem(x, e - 1, w)) r++;
    uint64_t len_off = 16, val_off = 16 + align16(4 * r);
    put_u32(out, (uint32_t)r);
    /* pass 2: emit each run */
    uint64_t run = 0, start = 0;
    for (uint64_t e = 1; e <= Fk; e++) {
        if (e == Fk || elem(x, e, w) != elem(x, e - 1, w)) {
            put_u32(out + len_off + 4 * run, (uint32_t)(e - start));
            put_elem(out + val_off, run, w, elem(x, start, w));
            run++;
            start = e;
        }
    }
    return val_off + align16(r * (uint64_t)w);
}

/* CSR — PAPER.md:220: "a non-zero value sequence and an additional index
 * representing the locations of non-zero values", (A00B0C000) -> (ABC),(035).
 * Rows of C elements (R5): u32 row_ptr[R+1] pad16 | u32 col_idx[nnz]
 * pad16 | values[nnz] pad16.                                                      */
static uint64_t enc_csr(const uint8_t* x, uint64_t Fk, int w, uint32_t C, uint8_t* out) {
    uint64_t R = ceil_div(Fk, C);
    uint64_t nnz_total = 0;
    for (uint64_t e = 0; e < Fk; e++) if (elem(x, e, w) != 0) nnz_total++;
    uint64_t rp_off = 0, ci_off = align16(4 * (R + 1)), v_off = ci_off + align16(4 * nnz_total);
    uint64_t nnz = 0;
    put_u32(out + rp_off, 0);
    for (uint64_t row = 0; row < R; row++) {
        for (uint64_t col = 0; col < C; col++) {
            uint64_t e = row * C + col;
            if (e >= Fk) break;
            uint32_t v = elem(x, e, w);
            if (v != 0) {
                put_u32(out + ci_off + 4 * nnz, (uint32_t)col);
                put_elem(out + v_off, nnz, w, v);
                nnz++;
            }
        }
        put_u32(out + rp_off + 4 * (row + 1), (uint32_t)nnz);
    }
    return v_off + align16(nnz * (uint64_t)w);
}

/* LZ4 — PAPER.md:220-222: "uses a dictionary-matching stage ... (abcde_bcde) can be
 * compressed as (abcde_(5,4))", [25] = nvcomp.  Output is the standard
 * LZ4 *block* format produced by the canonical greedy parse of DESIGN.md R6:
 * MINMATCH 4, MFLIMIT 12, LASTLITERALS 5, HASHLOG 12, lookup-then-insert at every
 * scanned position, no insertion inside matches, no skipping, no backward extension. */
#define LZ4_EMPTY 0xFFFFFFFFu

static uint32_t le32_at(const uint8_t* s, uint64_t i) { return get_u32(s + i); }

static uint64_t put_len_ext(uint8_t* out, uint64_t op, uint64_t v) {
    /* LZ4 length continuation: bytes of 255 then the remainder */
    while (v >= 255) { out[op++] = 255; v -= 255; }
    out[op++] = (uint8_t)v;
    return op;
}

static uint64_t lz4_emit(uint8_t* out, uint64_t op, const uint8_t* lit, uint64_t nlit,
                         int has_match, uint32_t offset, uint64_t mlen) {
    uint64_t tok_lit = nlit < 15 ? nlit : 15;
    uint64_t tok_m = 0;
    if (has_match) tok_m = (mlen - 4) < 15 ? (mlen - 4) : 15;
    out[op++] = (uint8_t)((tok_lit << 4) | tok_m);
    if (nlit >= 15) op = put_len_ext(out, op, nlit - 15);
    for (uint64_t i = 0; i < nlit; i++) out[op++] = lit[i];
    if (has_match) {
        put_u16(out + op, (uint16_t)offset);
        op += 2;
        if (mlen - 4 >= 15) op = put_len_ext(out, op, mlen - 4 - 15);
    }
    return op;
}

int64_t orc_lz4_block(const uint8_t* src, uint64_t L, uint8_t* out) {
    uint32_t T[4096]; /* hash table, starts EMPTY per block */
    for (int h = 0; h < 4096; h++) T[h] = LZ4_EMPTY;
    uint64_t anchor = 0, i = 0, op = 0;
    if (L >= 13) {
        while (i <= L - 12) {
            uint32_t h = (uint32_t)(le32_at(src, i) * 2654435761u) >> 20;
            uint32_t c = T[h];
            T[h] = (uint32_t)i; /* lookup, then insert */
            if (c != LZ4_EMPTY && le32_at(src, c) == le32_at(src, i)) {
                uint64_t len = 4;
                while (i + len < L - 5 && src[c + len] == src[i + len]) len++;
                op = lz4_emit(out, op, src + anchor, i - anchor, 1, (uint32_t)(i - c), len);
                i += len;
                anchor = i;
            } else {
                i += 1;
            }
        }
    }
    op = lz4_emit(out, op, src + anchor, L - anchor, 0, 0, 0);
    return (int64_t)op;
}

/* Standard LZ4 block decoder with full bounds checks; returns bytes written or <0. */
int64_t orc_lz4_block_decode(const uint8_t* in, uint64_t in_len, uint8_t* out, uint64_t out_cap) {
    uint64_t ip = 0, op = 0;
    for (;;) {
        if (ip >= in_len) return ORC_ERR_CORRUPT;
        uint32_t token = in[ip++];
        uint64_t nlit = token >> 4;
        if (nlit == 15) {
            uint32_t b;
            do {
                if (ip >= in_len) return ORC_ERR_CORRUPT;
                b = in[ip++];
                nlit += b;
            } while (b == 255);
        }
        if (ip + nlit > in_len || op + nlit > out_cap) return ORC_ERR_CORRUPT;
        for (uint64_t i = 0; i < nlit; i++) out[op++] = in[ip++];
        if (ip == in_len) return (int64_t)op; /* last sequence: literals only */
        if (ip + 2 > in_len) return ORC_ERR_CORRUPT;
        uint64_t offset = get_u16(in + ip);
        ip += 2;
        uint64_t mlen = (token & 15);
        if (mlen == 15) {
            uint32_t b;
            do {
                if (ip >= in_len) return ORC_ERR_CORRUPT;
                b = in[ip++];
                mlen += b;
            } while (b == 255);
        }
        mlen += 4;
        if (offset == 0 || offset > op || op + mlen > out_cap) return ORC_ERR_CORRUPT;
        for (uint64_t i = 0; i < mlen; i++) { out[op] = out[op - offset]; op++; } /* byte-wise: overlap-safe */
    }
}

static uint64_t lz4_block_bound(uint64_t L) { return L + L / 255 + 16; }

static uint64_t enc_lz4(const uint8_t* x, uint64_t Fk, int w, uint32_t B, uint8_t* out) {
    uint64_t bytes = Fk * (uint64_t)w;
    uint64_t nblk = ceil_div(bytes, B);
    uint64_t cs_off = 0, blk_off = align16(4 * nblk), op = blk_off;
    for (uint64_t b = 0; b < nblk; b++) {
        uint64_t s = b * B, L = bytes - s < B ? bytes - s : B;
        int64_t c = orc_lz4_block(x + s, L, out + op);
        put_u32(out + cs_off + 4 * b, (uint32_t)c);
        op += (uint64_t)c;
    }
    return align16(op);
}

/* ------------------------------------------------------------------------- */
/* Worst-case container size (capacity a caller must provide)                 */
/* ------------------------------------------------------------------------- */
uint64_t orc_max_size(int codec, int dtype, uint64_t n, uint64_t F, uint32_t param) {
    int w = width_of(dtype);
    if (w == 0 || F == 0) return 0;
    uint32_t K = (uint32_t)ceil_div(n, F);
    uint64_t total = data_start(K);
    for (uint64_t k = 0; k < K; k++) {
        uint64_t Fk = frame_elems(n, F, k);
        uint64_t raw = align16(Fk * (uint64_t)w);
        if (codec == C_NONE) total += raw;
        else if (codec == C_ZVC) total += align16(4 * ceil_div(Fk, 32)) + raw;
        else if (codec == C_RLE) total += 16 + align16(4 * Fk) + raw;
        else if (codec == C_CSR) total += align16(4 * (ceil_div(Fk, param) + 1)) + align16(4 * Fk) + raw;
        else if (codec == C_LZ4) {
            uint64_t bytes = Fk * (uint64_t)w, nblk = ceil_div(bytes, param), sum = 0;
            for (uint64_t b = 0; b < nblk; b++) {
                uint64_t L = bytes - b * param < param ? bytes - b * param : param;
                sum += lz4_block_bound(L);
            }
            total += align16(4 * nblk) + align16(sum);
        } else return 0;
    }
    return total;
}

static int params_ok(int codec, int dtype, uint64_t F, uint32_t param) {
    if (width_of(dtype) == 0) return 0;
    if (F == 0 || F % 1024 != 0) return 0;
    if (codec == C_CSR) return param > 0 && F % param == 0;
    if (codec == C_LZ4) return param > 0 && param <= 65536 && param % 1024 == 0;
    if (codec == C_NONE || codec == C_ZVC || codec == C_RLE) return param == 0;
    return 0;
}

/* Compress n elements into a canonical container v1.  Returns the container size
 * or a negative ORC_ERR_*.  `out` must hold `cap` bytes. */
int64_t orc_compress(int codec, int dtype, const void* in, uint64_t n, uint64_t F, uint32_t param,
                     void* out_v, uint64_t cap) {
    if (!params_ok(codec, dtype, F, param)) return ORC_ERR_INVALID;
    int w = width_of(dtype);
    uint64_t need = orc_max_size(codec, dtype, n, F, param);
    if (cap < need) return ORC_ERR_CAPACITY;
    uint8_t* out = (uint8_t*)out_v;
    const uint8_t* x = (const uint8_t*)in;
    memset(out, 0, need);
    uint32_t K = (uint32_t)ceil_div(n, F);
    uint64_t pos = data_start(K);
    for (uint64_t k = 0; k < K; k++) {
        uint64_t Fk = frame_elems(n, F, k);
        const uint8_t* xf = x + k * F * (uint64_t)w;
        uint64_t fb = 0;
        if (codec == C_NONE) fb = enc_none(xf, Fk, w, out + pos);
        else if (codec == C_ZVC) fb = enc_zvc(xf, Fk, w, out + pos);
        else if (codec == C_RLE) fb = enc_rle(xf, Fk, w, out + pos);
        else if (codec == C_CSR) fb = enc_csr(xf, Fk, w, param, out + pos);
        else fb = enc_lz4(xf, Fk, w, param, out + pos);
        put_u64(out + 64 + 8 * k, fb);
        pos += fb;
    }
    memcpy(out, "CSWP", 4);
    put_u16(out + 4, 1);
    out[6] = (uint8_t)codec;
    out[7] = (uint8_t)dtype;
    put_u64(out + 8, n);
    put_u64(out + 16, F);
    put_u32(out + 24, K);
    put_u32(out + 28, param);
    put_u64(out + 32, pos);
    /* bytes [pos, need) were zeroed above and are not part of the container */
    return (int64_t)pos;
}

/* ------------------------------------------------------------------------- */
/* Decoders (validate everything; never read or write out of bounds)          */
/* ------------------------------------------------------------------------- */
static int dec_frame(int codec, int w, uint32_t param, const uint8_t* p, uint64_t fb, uint64_t Fk,
                     uint8_t* y) {
    if (fb % 16 != 0) return ORC_ERR_CORRUPT;
    if (codec == C_NONE) {
        if (fb != align16(Fk * (uint64_t)w)) return ORC_ERR_CORRUPT;
        memcpy(y, p, Fk * (uint64_t)w);
        return ORC_OK;
    }
    if (codec == C_ZVC) {
        /* dense[i] = bit(i) ? values[#set bits before i] : 0 */
        uint64_t nwords = ceil_div(Fk, 32), bm = align16(4 * nwords);
        if (fb < bm) return ORC_ERR_CORRUPT;
        uint64_t rank = 0;
        for (uint64_t e = 0; e < nwords * 32; e++) {
            uint32_t word = get_u32(p + 4 * (e / 32));
            int bit = (word >> (e % 32)) & 1;
            if (e >= Fk) { if (bit) return ORC_ERR_CORRUPT; continue; }
            if (bit) {
                if (bm + (rank + 1) * (uint64_t)w > fb) return ORC_ERR_CORRUPT;
                put_elem(y, e, w, elem(p + bm, rank, w));
                rank++;
            } else {
                put_elem(y, e, w, 0);
            }
        }
        if (fb != bm + align16(rank * (uint64_t)w)) return ORC_ERR_CORRUPT;
        return ORC_OK;
    }
    if (codec == C_RLE) {
        if (fb < 16) return ORC_ERR_CORRUPT;
        uint64_t r = get_u32(p);
        if (r == 0 || r > Fk) return ORC_ERR_CORRUPT;
        uint64_t len_off = 16, val_off = 16 + align16(4 * r);
        if (fb != val_off + align16(r * (uint64_t)w)) return ORC_ERR_CORRUPT;
        uint64_t e = 0;
        for (uint64_t run = 0; run < r; run++) {
            uint64_t L = get_u32(p + len_off + 4 * run);
            if (L == 0 || e + L > Fk) return ORC_ERR_CORRUPT;
            uint32_t v = elem(p + val_off, run, w);
            for (uint64_t i = 0; i < L; i++) put_elem(y, e + i, w, v);
            e += L;
        }
        if (e != Fk) return ORC_ERR_CORRUPT;
        return ORC_OK;
    }
    if (codec == C_CSR) {
        uint64_t C = param, R = ceil_div(Fk, C);
        uint64_t ci_off = align16(4 * (R + 1));
        if (fb < ci_off) return ORC_ERR_CORRUPT;
        uint64_t nnz = get_u32(p + 4 * R);
        if (get_u32(p) != 0 || nnz > Fk) return ORC_ERR_CORRUPT;
        uint64_t v_off = ci_off + align16(4 * nnz);
        if (fb != v_off + align16(nnz * (uint64_t)w)) return ORC_ERR_CORRUPT;
        memset(y, 0, Fk * (uint64_t)w); /* zero-fill, then scatter */
        for (uint64_t row = 0; row < R; row++) {
            uint64_t a = get_u32(p + 4 * row), b = get_u32(p + 4 * (row + 1));
            uint64_t width = (row + 1) * C <= Fk ? C : Fk - row * C;
            if (b < a || b > nnz) return ORC_ERR_CORRUPT;
            for (uint64_t q = a; q < b; q++) {
                uint64_t col = get_u32(p + ci_off + 4 * q);
                if (col >= width) return ORC_ERR_CORRUPT;
                if (q > a && col <= get_u32(p + ci_off + 4 * (q - 1))) return ORC_ERR_CORRUPT;
                put_elem(y, row * C + col, w, elem(p + v_off, q, w));
            }
        }
        return ORC_OK;
    }
    if (codec == C_LZ4) {
        uint64_t bytes = Fk * (uint64_t)w, B = param, nblk = ceil_div(bytes, B);
        uint64_t cs_off = 0, op = align16(4 * nblk);
        if (fb < op) return ORC_ERR_CORRUPT;
        for (uint64_t b = 0; b < nblk; b++) {
            uint64_t cs = get_u32(p + cs_off + 4 * b);
            uint64_t L = bytes - b * B < B ? bytes - b * B : B;
            if (op + cs > fb) return ORC_ERR_CORRUPT;
            int64_t got = orc_lz4_block_decode(p + op, cs, y + b * B, L);
            if (got != (int64_t)L) return ORC_ERR_CORRUPT;
            op += cs;
        }
        if (fb != align16(op)) return ORC_ERR_CORRUPT;
        return ORC_OK;
    }
    return ORC_ERR_CORRUPT;
}

/* Decompress a container into n elements of dtype.  0 on success, <0 on error. */
int orc_decompress(const void* in_v, uint64_t in_size, void* out_v, uint64_t n, int dtype) {
    const uint8_t* in = (const uint8_t*)in_v;
    if (in_size < 64) return ORC_ERR_CORRUPT;
    if (memcmp(in, "CSWP", 4) != 0 || get_u16(in + 4) != 1) return ORC_ERR_CORRUPT;
    int codec = in[6], dt = in[7];
    uint64_t hn = get_u64(in + 8), F = get_u64(in + 16), total = get_u64(in + 32);
    uint32_t K = get_u32(in + 24), param = get_u32(in + 28);
    if (dt != dtype || hn != n) return ORC_ERR_INVALID;
    if (!params_ok(codec, dtype, F, param)) return ORC_ERR_CORRUPT;
    if ((uint64_t)K != ceil_div(n, F)) return ORC_ERR_CORRUPT;
    if (total > in_size || data_start(K) > total) return ORC_ERR_CORRUPT;
    int w = width_of(dtype);
    uint64_t pos = data_start(K);
    for (uint64_t k = 0; k < K; k++) {
        uint64_t fb = get_u64(in + 64 + 8 * k);
        if (fb > total - pos) return ORC_ERR_CORRUPT;
        int rc = dec_frame(codec, w, param, in + pos, fb, frame_elems(n, F, k),
                           (uint8_t*)out_v + k * F * (uint64_t)w);
        if (rc != ORC_OK) return rc;
        pos += fb;
    }
    if (pos != total) return ORC_ERR_CORRUPT;
    return ORC_OK;
}

/* ------------------------------------------------------------------------- */
/* Sparsity probe — PAPER.md:118 (§IV-A, "collects ... sparsity"), :327 (§V-E,  */
/* "CSWAP utilizes GPU multi-cores to profile tensor sparsity"), Table II       */
/* Sparsity^t (:131).  Deterministic windows, R15.                    */
/* counts = {zeros, zero_runs, boundaries, samples, pairs}                     */
/* ------------------------------------------------------------------------- */
#define PROBE_W 256
#define PROBE_SW 1024

void orc_probe(const void* in, uint64_t n, int dtype, uint64_t counts[5]) {
    const uint8_t* x = (const uint8_t*)in;
    int w = width_of(dtype);
    for (int c = 0; c < 5; c++) counts[c] = 0;
    if (n == 0 || w == 0) return;
    uint64_t nwin = n <= (uint64_t)PROBE_SW * PROBE_W ? 1 : PROBE_SW;
    for (uint64_t k = 0; k < nwin; k++) {
        uint64_t start, len;
        if (nwin == 1) { start = 0; len = n; }
        else { start = k * (n - PROBE_W) / (PROBE_SW - 1); len = PROBE_W; }
        for (uint64_t i = start; i < start + len; i++) {
            uint32_t v = elem(x, i, w);
            if (v == 0) counts[0]++;
            if (v == 0 && (i == start || elem(x, i - 1, w) != 0)) counts[1]++;
            if (i > start && v != elem(x, i - 1, w)) counts[2]++;
        }
        counts[3] += len;
        counts[4] += len - 1;
    }
}

/* Integer estimates (u64, round-half-up, no floating point — DESIGN.md R19).
 * est = {zeros_hat, nnz_hat, runs_hat, zero_runs_hat} */
void orc_probe_estimates(uint64_t n, const uint64_t counts[5], uint64_t est[4]) {
    uint64_t zeros = counts[0], zruns = counts[1], bnd = counts[2], samples = counts[3], pairs = counts[4];
    if (samples == 0) { est[0] = est[1] = 0; est[2] = n ? 1 : 0; est[3] = 0; return; }
    est[0] = (zeros * n + samples / 2) / samples;
    est[1] = n - est[0];
    est[2] = pairs == 0 ? 1 : 1 + (bnd * (n - 1) + pairs / 2) / pairs;
    est[3] = (zruns * n + samples / 2) / samples;
}

/* ------------------------------------------------------------------------- */
/* Selector — PAPER.md:137-154 (§IV-B, Eq. 1-4) and :30 (pick one of four).     */
/* Plain double arithmetic in the order written.  DESIGN.md R8-R14, R20.       */
/* ------------------------------------------------------------------------- */
typedef struct {
    double alpha_d2h, bw_d2h, alpha_h2d, bw_h2d;   /* link: t = alpha + bytes / bw  (s, B/s) */
    double beta[4][2][6][3];                        /* [codec-1][0=c,1=dc][band][b0,b1,b2]: t = b0 + b1*S + b2*S*s */
    double lz4_gamma1, lz4_gamma2;
    double margin;                                  /* pipelined mode only */
    int32_t mode;                                   /* 0 = pipelined (default), 1 = paper */
    int32_t pad_;
    uint64_t frame_elems;                           /* F */
    uint32_t csr_row, lz4_block;                    /* C, B */
    double group_bytes;                             /* swap-in pipeline step (R22) */
} orc_calib;

static int band_of(double s) {
    /* bands [0,.2) [.2,.35) [.35,.5) [.5,.65) [.65,.8) [.8,1]  (R14) */
    if (s < 0.2) return 0;
    if (s < 0.35) return 1;
    if (s < 0.5) return 2;
    if (s < 0.65) return 3;
    if (s < 0.8) return 4;
    return 5;
}

static double dmax(double a, double b) { return a > b ? a : b; }
static double dmin(double a, double b) { return a < b ? a : b; }

/* out: [0]=codec chosen, [1]=T(c*), [2]=T', [3..6]=T(ZVC..LZ4), [7..10]=predicted bytes,
 *      [11..14]=t_c, [15..18]=t_dc */
int orc_select(uint64_t n, int dtype, const uint64_t counts[5], double hidden_f, double hidden_b,
               const orc_calib* cal, double out[19]) {
    int w = width_of(dtype);
    for (int i = 0; i < 19; i++) out[i] = 0;
    if (w == 0) return ORC_ERR_INVALID;
    if (n == 0 || counts[3] == 0) { out[0] = C_NONE; return ORC_OK; }
    uint64_t est[4];
    orc_probe_estimates(n, counts, est);
    double S = (double)n * (double)w;
    double s = (double)counts[0] / (double)counts[3];
    int band = band_of(s);
    int paper = cal->mode == 1;
    double a_d2h = paper ? 0.0 : cal->alpha_d2h;
    double a_h2d = paper ? 0.0 : cal->alpha_h2d;
    uint64_t F = cal->frame_elems;
    uint64_t K = ceil_div(n, F);

    /* Eq. 1: T' = max(S/BW_d2h - Hf, 0) + max(S/BW_h2d - Hb, 0) */
    double Tp = dmax(a_d2h + S / cal->bw_d2h - hidden_f, 0.0) + dmax(a_h2d + S / cal->bw_h2d - hidden_b, 0.0);

    double best = 0;
    int best_c = 0;
    for (int c = 1; c <= 4; c++) {
        const double* bc = cal->beta[c - 1][0][band];
        const double* bd = cal->beta[c - 1][1][band];
        double tc = bc[0] + bc[1] * S + bc[2] * S * s;
        double tdc = bd[0] + bd[1] * S + bd[2] * S * s;
        double size;
        if (paper) {
            size = S * (1.0 - s); /* Eq. 3-4: Size x (1 - Sparsity) */
        } else {
            uint64_t hdr = data_start((uint32_t)K), fixed = 0;
            for (uint64_t k = 0; k < K; k++) {
                uint64_t Fk = frame_elems(n, F, k);
                if (c == C_ZVC) fixed += align16(4 * ceil_div(Fk, 32));
                if (c == C_CSR) fixed += align16(4 * (ceil_div(Fk, cal->csr_row) + 1));
                if (c == C_RLE) fixed += 16;
                if (c == C_LZ4) fixed += align16(4 * ceil_div(Fk * (uint64_t)w, cal->lz4_block));
            }
            if (c == C_ZVC) {
                size = (double)(hdr + fixed + align16(est[1] * (uint64_t)w));
            } else if (c == C_CSR) {
                size = (double)(hdr + fixed + align16(4 * est[1]) + align16(est[1] * (uint64_t)w));
            } else if (c == C_RLE) {
                uint64_t r = est[2] + (K - 1);
                if (r > n) r = n;
                size = (double)(hdr + fixed + align16(4 * r) + align16(r * (uint64_t)w));
            } else {
                size = (double)(hdr + fixed) + (double)(est[1] * (uint64_t)w) +
                       cal->lz4_gamma1 * (double)est[3] + cal->lz4_gamma2 * (double)w * (double)est[0] / 255.0;
            }
        }
        double xo = a_d2h + size / cal->bw_d2h;
        double xi = a_h2d + size / cal->bw_h2d;
        double T;
        if (paper) {
            /* Eq. 2: T = Time_c + Time_dc + O_f + O_b */
            T = tc + tdc + dmax(xo - hidden_f, 0.0) + dmax(xi - hidden_b, 0.0);
        } else {
            /* pipelined mode models the executor it predicts (R11, R22).
             * Swap-out: ZVC hands every finished frame to the copy engine while later frames
             * are compressed -> a K-step pipeline; RLE, CSR and LZ4 place a frame only after
             * every frame has been counted / parsed -> codec time then transfer. */
            double Tout;
            if (c == C_ZVC)
                Tout = dmax(tc, xo) + dmin(tc, xo) / (double)K;
            else
                Tout = tc + xo;
            /* Swap-in: H2D + decode in groups of whole frames of >= group_bytes container
             * bytes: G = ceil(K / q), q = ceil(group_bytes / frame bytes), frames of equal
             * size (size - header) / K; group_bytes <= 0 -> one frame per step (G = K). */
            double G = (double)K;
            double sf = (size - (double)data_start((uint32_t)K)) / (double)K;
            if (cal->group_bytes > 0 && sf > 0) {
                double q = ceil(cal->group_bytes / sf);
                G = ceil((double)K / q);
            }
            double Tin = dmax(tdc, xi) + dmin(tdc, xi) / G;
            T = dmax(Tout - hidden_f, 0.0) + dmax(Tin - hidden_b, 0.0);
        }
        out[3 + c - 1] = T;
        out[7 + c - 1] = size;
        out[11 + c - 1] = tc;
        out[15 + c - 1] = tdc;
        if (c == 1 || T < best) { best = T; best_c = c; } /* ties -> lower codec id */
    }
    double m = paper ? 0.0 : cal->margin;
    out[1] = best;
    out[2] = Tp;
    /* "If T' > T, a compression plan ... is generated; otherwise, no compression" */
    out[0] = best < (1.0 - m) * Tp ? best_c : C_NONE;
    return ORC_OK;
}

/* ------------------------------------------------------------------------- */
/* Relative absolute error — PAPER.md:301 (§V-C):                              */
/*   RAE = sum|yhat_i - y_i| / sum|ybar - y_i|                                   */
/* ------------------------------------------------------------------------- */
double orc_rae(const double* yhat, const double* y, uint64_t N) {
    double mean = 0;
    for (uint64_t i = 0; i < N; i++) mean += y[i];
    mean /= (double)N;
    double num = 0, den = 0;
    for (uint64_t i = 0; i < N; i++) {
        num += yhat[i] > y[i] ? yhat[i] - y[i] : y[i] - yhat[i];
        den += mean > y[i] ? mean - y[i] : y[i] - mean;
    }
    return num / den;
}
