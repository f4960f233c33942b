/*
 * cszp2_oracle.c — plain single-threaded CPU oracle (TEST INFRASTRUCTURE ONLY).
 * See cszp2_oracle.h for the scope and FORMAT.md for the contract it follows.
 * Build: gcc -std=c11 -O2 -ffp-contract=off -fno-fast-math (no FMA, SSE2 scalar).
 */
#include "cszp2_oracle.h"

#include <math.h>
#include <stdlib.h>
#include <string.h>

#define BPT 256u               /* blocks per tile (FORMAT.md §1) */
#define MAGIC 0x325A5343u      /* "CSZ2" */

/* ---------- small helpers (obvious by inspection) ---------- */

static uint64_t roundup16(uint64_t v) { return (v + 15u) / 16u * 16u; }

/* number of significant bits of v; 0 for 0 (FORMAT.md §6.5) */
static int bitlen(uint32_t v) {
    int n = 0;
    while (v != 0) {
        n++;
        v >>= 1;
    }
    return n;
}

static int log2_of(int L) {
    int k = 0;
    while ((1 << k) < L) k++;
    return k;
}

static int valid_L(int L) { return L == 8 || L == 32 || L == 64; }

static void put_u16(uint8_t *p, uint16_t v) {
    p[0] = (uint8_t)(v & 0xFF);
    p[1] = (uint8_t)(v >> 8);
}
static void put_u32(uint8_t *p, uint32_t v) {
    for (int i = 0; i < 4; i++) p[i] = (uint8_t)(v >> (8 * i));
}
static void put_u64(uint8_t *p, uint64_t v) {
    for (int i = 0; i < 8; i++) p[i] = (uint8_t)(v >> (8 * i));
}
static void put_f64(uint8_t *p, double v) {
    uint64_t u;
    memcpy(&u, &v, 8);
    put_u64(p, u);
}
static uint16_t get_u16(const uint8_t *p) { return (uint16_t)(p[0] | (p[1] << 8)); }
static uint32_t get_u32(const uint8_t *p) {
    uint32_t v = 0;
    for (int i = 3; i >= 0; i--) v = (v << 8) | p[i];
    return v;
}
static uint64_t get_u64(const uint8_t *p) {
    uint64_t v = 0;
    for (int i = 7; i >= 0; i--) v = (v << 8) | p[i];
    return v;
}
static double get_f64(const uint8_t *p) {
    uint64_t u = get_u64(p);
    double v;
    memcpy(&v, &u, 8);
    return v;
}

/* set / get bit i of an L-bit field stored LSB-first (FORMAT.md §5) */
static void field_set(uint8_t *field, int i) { field[i / 8] |= (uint8_t)(1u << (i % 8)); }
static int field_get(const uint8_t *field, int i) { return (field[i / 8] >> (i % 8)) & 1; }

/* ---------- stream geometry (FORMAT.md §2) ---------- */

typedef struct {
    uint64_t nb, T, O, D;
} geom_t;

static geom_t geometry(uint64_t n, int L) {
    geom_t g;
    g.nb = (n + (uint64_t)L - 1) / (uint64_t)L;
    g.T = (g.nb + BPT - 1) / BPT;
    g.O = roundup16(64 + 8 * g.T);
    g.D = roundup16(g.O + g.nb);
    return g;
}

uint64_t oracle_compress_bound(uint64_t n, int L) {
    geom_t g = geometry(n, L);
    return roundup16(g.D + (uint64_t)(4 * L) * g.nb);
}

/* ---------- step 0: error bound (FORMAT.md §6.1) ---------- */

int oracle_resolve_eb(const void *x, uint64_t n, int dtype, double eb, int eb_mode,
                      double *eb_abs) {
    if (!(eb > 0.0) || !isfinite(eb)) return ORC_ERR_ARG;
    if (eb_mode == ORC_ABS) {
        *eb_abs = eb;
        return ORC_OK;
    }
    if (eb_mode != ORC_REL) return ORC_ERR_ARG;
    int have = 0;
    double r = 0.0;
    if (dtype == ORC_F32) {
        const float *v = (const float *)x;
        float mn = 0.0f, mx = 0.0f;
        for (uint64_t i = 0; i < n; i++) {
            float a = v[i];
            if (isnan(a)) continue;
            if (!have) {
                mn = a;
                mx = a;
                have = 1;
            }
            if (a < mn) mn = a;
            if (a > mx) mx = a;
        }
        if (have) r = (double)mx - (double)mn;
    } else {
        const double *v = (const double *)x;
        double mn = 0.0, mx = 0.0;
        for (uint64_t i = 0; i < n; i++) {
            double a = v[i];
            if (isnan(a)) continue;
            if (!have) {
                mn = a;
                mx = a;
                have = 1;
            }
            if (a < mn) mn = a;
            if (a > mx) mx = a;
        }
        if (have) r = mx - mn;
    }
    if (r == 0.0)
        *eb_abs = eb;
    else
        *eb_abs = eb * r;
    return ORC_OK;
}

/* FORMAT.md §6.2: are the constants derived from eb_abs usable? */
static int constants_ok(int dtype, double eb_abs) {
    if (!(eb_abs > 0.0) || !isfinite(eb_abs)) return 0;
    if (dtype == ORC_F32) {
        float inv = (float)(1.0 / (2.0 * eb_abs));
        float s = (float)(2.0 * eb_abs);
        return inv > 0.0f && isfinite(inv) && s > 0.0f && isfinite(s);
    }
    double inv = 1.0 / (2.0 * eb_abs);
    double s = 2.0 * eb_abs;
    return inv > 0.0 && isfinite(inv) && s > 0.0 && isfinite(s);
}

/* ---------- step ❶: lossy conversion (FORMAT.md §6.3) ---------- */

/* FORMAT.md §6.3 / §7: largest accepted |t| per predictor (1D, 2D, 3D) */
static const float TMAX_F32[3] = {1073741760.0f, 268435440.0f, 134217720.0f};
static const double TMAX_F64[3] = {1073741823.0, 268435455.0, 134217727.0};

static int quantize_p(const void *x, uint64_t n, int dtype, double eb_abs, int32_t *q, int pred) {
    int status = ORC_OK;
    if (!constants_ok(dtype, eb_abs)) status = ORC_ERR_RANGE;
    if (dtype == ORC_F32) {
        const float *v = (const float *)x;
        float inv = (float)(1.0 / (2.0 * eb_abs));
        for (uint64_t i = 0; i < n; i++) {
            float t = v[i] * inv; /* one RN multiply in f32 */
            if (!(fabsf(t) <= TMAX_F32[pred])) {
                status = ORC_ERR_RANGE;
                q[i] = 0;
                continue;
            }
            q[i] = (int32_t)nearbyintf(t); /* ties to even in FE_TONEAREST */
        }
    } else {
        const double *v = (const double *)x;
        double inv = 1.0 / (2.0 * eb_abs);
        for (uint64_t i = 0; i < n; i++) {
            double t = v[i] * inv;
            if (!(fabs(t) <= TMAX_F64[pred])) {
                status = ORC_ERR_RANGE;
                q[i] = 0;
                continue;
            }
            q[i] = (int32_t)nearbyint(t);
        }
    }
    return status;
}

int oracle_quantize(const void *x, uint64_t n, int dtype, double eb_abs, int32_t *q) {
    return quantize_p(x, n, dtype, eb_abs, q, 0);
}

void oracle_dequantize(const int32_t *q, uint64_t n, int dtype, double eb_abs, void *x) {
    if (dtype == ORC_F32) {
        float s = (float)(2.0 * eb_abs);
        float *o = (float *)x;
        for (uint64_t i = 0; i < n; i++) o[i] = (float)q[i] * s;
    } else {
        double s = 2.0 * eb_abs;
        double *o = (double *)x;
        for (uint64_t i = 0; i < n; i++) o[i] = (double)q[i] * s;
    }
}

/* ---------- step ❷: first-order difference + FLE ---------- */

/* ❷ FLE of one block of L residuals d: offset byte + payload; returns
 * the payload size. */
static int fle_encode(const int32_t *d, int L, int enc_mode, uint8_t *offset_byte,
                      uint8_t *payload) {
    uint32_t a[64];
    int fb = L / 8; /* bytes per bit field */
    for (int i = 0; i < L; i++) a[i] = (uint32_t)(d[i] < 0 ? -(int64_t)d[i] : (int64_t)d[i]);

    /* Plain-FLE statistics */
    uint32_t or_all = 0;
    for (int i = 0; i < L; i++) or_all |= a[i];
    int fl_p = bitlen(or_all);
    int size_p = fl_p ? fb * (1 + fl_p) : 0;

    /* Outlier-FLE statistics and the fine-tuned selection */
    int use_outlier = 0, fl_o = 0, ob = 0, size_o = 0;
    if (enc_mode == ORC_OUTLIER) {
        uint32_t or_rest = 0;
        for (int i = 1; i < L; i++) or_rest |= a[i];
        fl_o = bitlen(or_rest);
        ob = (bitlen(a[0]) + 7) / 8;
        if (ob < 1) ob = 1;
        size_o = fb + ob + fb * fl_o;
        use_outlier = size_o < size_p;
    }

    int pos = 0;
    if (!use_outlier) {
        *offset_byte = (uint8_t)fl_p;
        if (fl_p == 0) return 0;
        memset(payload, 0, (size_t)size_p);
        for (int i = 0; i < L; i++)
            if (d[i] < 0) field_set(payload, i);
        pos = fb;
        for (int k = 0; k < fl_p; k++) {
            for (int i = 0; i < L; i++)
                if ((a[i] >> k) & 1u) field_set(payload + pos, i);
            pos += fb;
        }
        return size_p;
    }

    *offset_byte = (uint8_t)(0x80 | ((ob - 1) << 5) | fl_o);
    memset(payload, 0, (size_t)size_o);
    for (int i = 0; i < L; i++)
        if (d[i] < 0) field_set(payload, i);
    pos = fb;
    for (int j = 0; j < ob; j++) payload[pos + j] = (uint8_t)(a[0] >> (8 * j));
    pos += ob;
    for (int k = 0; k < fl_o; k++) {
        for (int i = 1; i < L; i++)
            if ((a[i] >> k) & 1u) field_set(payload + pos, i);
        pos += fb;
    }
    return size_o;
}

int oracle_encode_block(const int32_t *q, int L, int enc_mode, uint8_t *offset_byte,
                        uint8_t *payload) {
    int32_t d[64];
    /* first-order difference inside the block, q_{-1} = 0 (FORMAT.md §6.4) */
    for (int i = 0; i < L; i++) {
        int32_t prev = (i == 0) ? 0 : q[i - 1];
        d[i] = (int32_t)((int64_t)q[i] - (int64_t)prev);
    }
    return fle_encode(d, L, enc_mode, offset_byte, payload);
}

int oracle_block_size(uint8_t ob_byte, int L) {
    int fb = L / 8;
    int fl = ob_byte & 31;
    if (ob_byte & 0x80) {
        int ob = ((ob_byte >> 5) & 3) + 1;
        return fb + ob + fb * fl;
    }
    if (ob_byte & 0x60) return -1;
    return fl ? fb * (1 + fl) : 0;
}

/* ❷⁻¹: residuals of one block from its offset byte + payload (size or -1) */
static int fle_decode(uint8_t ob_byte, const uint8_t *payload, int L, int32_t *d) {
    int fb = L / 8;
    int size = oracle_block_size(ob_byte, L);
    if (size < 0) return -1;
    uint32_t a[64];
    for (int i = 0; i < L; i++) a[i] = 0;
    int fl = ob_byte & 31;
    if (size > 0) {
        const uint8_t *signs = payload;
        int pos = fb;
        int first = 0;
        if (ob_byte & 0x80) {
            int ob = ((ob_byte >> 5) & 3) + 1;
            uint32_t v = 0;
            for (int j = ob - 1; j >= 0; j--) v = (v << 8) | payload[pos + j];
            a[0] = v;
            pos += ob;
            first = 1;
        }
        for (int k = 0; k < fl; k++) {
            for (int i = first; i < L; i++)
                if (field_get(payload + pos, i)) a[i] |= (1u << k);
            pos += fb;
        }
        for (int i = 0; i < L; i++)
            d[i] = field_get(signs, i) ? -(int32_t)a[i] : (int32_t)a[i];
    } else {
        for (int i = 0; i < L; i++) d[i] = 0;
    }
    return size;
}

int oracle_decode_block(uint8_t ob_byte, const uint8_t *payload, int L, int32_t *q) {
    int32_t d[64];
    int size = fle_decode(ob_byte, payload, L, d);
    if (size < 0) return -1;
    /* inverse first-order difference, q_{-1} = 0 (FORMAT.md §6.6) */
    int32_t prev = 0;
    for (int i = 0; i < L; i++) {
        prev = (int32_t)((uint32_t)prev + (uint32_t)d[i]);
        q[i] = prev;
    }
    return size;
}

/* ---------- steps ❸ + ❹: serial prefix sum and concatenation ---------- */

/* Encode nb blocks of given (already quantized) integers into `out` following
 * FORMAT.md §2; header fields other than geometry are filled by the caller. */
static void encode_stream(const int32_t *q, uint64_t n, int enc_mode, int L, uint8_t *out,
                          uint64_t *payload_bytes, uint64_t *total) {
    geom_t g = geometry(n, L);
    uint8_t *offsets = out + g.O;
    uint8_t *payloads = out + g.D;
    int32_t blk[64];
    uint8_t buf[4 * 64 + 8];
    uint64_t excl = 0; /* exclusive prefix of payload sizes: a plain loop */

    memset(out, 0, (size_t)g.D);
    for (uint64_t b = 0; b < g.nb; b++) {
        for (int i = 0; i < L; i++) {
            uint64_t idx = b * (uint64_t)L + (uint64_t)i;
            if (idx < n)
                blk[i] = q[idx];
            else
                blk[i] = blk[i - 1]; /* tail padding, FORMAT.md §6.4 */
        }
        uint8_t ob_byte = 0;
        int size = oracle_encode_block(blk, L, enc_mode, &ob_byte, buf);
        offsets[b] = ob_byte;
        memcpy(payloads + excl, buf, (size_t)size);
        excl += (uint64_t)size;
        /* tile index: inclusive sum at the end of each tile */
        if ((b + 1) % BPT == 0 || b + 1 == g.nb) {
            uint64_t t = b / BPT;
            put_u64(out + 64 + 8 * t, (2ull << 62) | excl);
        }
    }
    uint64_t tot = roundup16(g.D + excl);
    memset(payloads + excl, 0, (size_t)(tot - g.D - excl));
    *payload_bytes = excl;
    *total = tot;
}

static void write_header(uint8_t *out, int dtype, int enc_mode, int L, int eb_mode, int status,
                         uint64_t n, double eb, double eb_abs, uint64_t pb, uint64_t total) {
    memset(out, 0, 64);
    put_u32(out + 0, MAGIC);
    out[4] = 1;
    out[5] = (uint8_t)dtype;
    out[6] = (uint8_t)enc_mode;
    out[7] = (uint8_t)log2_of(L);
    out[8] = (uint8_t)eb_mode;
    out[9] = (uint8_t)status;
    put_u16(out + 10, (uint16_t)BPT);
    put_u64(out + 16, n);
    put_f64(out + 24, eb);
    put_f64(out + 32, eb_abs);
    put_u64(out + 40, pb);
    put_u64(out + 48, total);
}

int oracle_compress(const void *x, uint64_t n, int dtype, double eb, int eb_mode,
                    int enc_mode, int L, uint8_t *out, uint64_t *out_bytes) {
    if (!valid_L(L) || (dtype != ORC_F32 && dtype != ORC_F64) ||
        (enc_mode != ORC_PLAIN && enc_mode != ORC_OUTLIER) || (!x && n))
        return ORC_ERR_ARG;
    double eb_abs = 0.0;
    int rc = oracle_resolve_eb(x, n, dtype, eb, eb_mode, &eb_abs);
    if (rc != ORC_OK) return rc;

    int32_t *q = (int32_t *)malloc((size_t)(n ? n : 1) * sizeof(int32_t));
    if (!q) return ORC_ERR_ARG;
    int status = oracle_quantize(x, n, dtype, eb_abs, q);
    uint64_t pb = 0, total = 0;
    if (status == ORC_OK) {
        encode_stream(q, n, enc_mode, L, out, &pb, &total);
    } else {
        /* RANGE: only the header is specified (FORMAT.md §6.7); emit it alone */
        geom_t g = geometry(n, L);
        pb = 0;
        total = roundup16(g.D);
        memset(out, 0, (size_t)total);
    }
    free(q);
    write_header(out, dtype, enc_mode, L, eb_mode, status, n, eb, eb_abs, pb, total);
    *out_bytes = total;
    return status;
}

int oracle_compress_ints(const int32_t *q, uint64_t n, int enc_mode, int L, uint8_t *out,
                         uint64_t *out_bytes) {
    if (!valid_L(L) || (enc_mode != ORC_PLAIN && enc_mode != ORC_OUTLIER)) return ORC_ERR_ARG;
    for (uint64_t i = 0; i < n; i++)
        if (q[i] > 1073741823 || q[i] < -1073741823) return ORC_ERR_ARG;
    uint64_t pb = 0, total = 0;
    encode_stream(q, n, enc_mode, L, out, &pb, &total);
    write_header(out, ORC_F32, enc_mode, L, ORC_ABS, ORC_OK, n, 0.0, 0.0, pb, total);
    *out_bytes = total;
    return ORC_OK;
}

/* ---------- decompression: ❸ locate → ❹ → ❷⁻¹ → ❶⁻¹ ---------- */

static int decode_stream(const uint8_t *cmp, uint64_t cmp_bytes, uint64_t n, int32_t *q,
                         int *L_out) {
    if (cmp_bytes < 64) return ORC_ERR_FORMAT;
    if (get_u32(cmp) != MAGIC || cmp[4] != 1) return ORC_ERR_FORMAT;
    int log2L = cmp[7];
    if (log2L != 3 && log2L != 5 && log2L != 6) return ORC_ERR_FORMAT;
    int L = 1 << log2L;
    *L_out = L;
    if (get_u16(cmp + 10) != BPT) return ORC_ERR_FORMAT;
    if (cmp[12] != 0) return ORC_ERR_FORMAT; /* a multi-dimensional stream (FORMAT.md §7) */
    if (get_u64(cmp + 16) != n) return ORC_ERR_FORMAT;
    if (cmp[9] == ORC_ERR_RANGE) return ORC_ERR_RANGE;
    if (cmp[9] != 0) return ORC_ERR_FORMAT;
    geom_t g = geometry(n, L);
    uint64_t pb = get_u64(cmp + 40), total = get_u64(cmp + 48);
    if (total != roundup16(g.D + pb) || total > cmp_bytes) return ORC_ERR_FORMAT;

    const uint8_t *offsets = cmp + g.O;
    const uint8_t *payloads = cmp + g.D;
    uint64_t excl = 0; /* serial prefix sum of sizes read from the offset bytes */
    int32_t blk[64];
    for (uint64_t b = 0; b < g.nb; b++) {
        int size = oracle_block_size(offsets[b], L);
        if (size < 0 || excl + (uint64_t)size > pb) return ORC_ERR_FORMAT;
        oracle_decode_block(offsets[b], payloads + excl, L, blk);
        excl += (uint64_t)size;
        for (int i = 0; i < L; i++) {
            uint64_t idx = b * (uint64_t)L + (uint64_t)i;
            if (idx < n) q[idx] = blk[i];
        }
        if ((b + 1) % BPT == 0 || b + 1 == g.nb) {
            uint64_t t = b / BPT;
            if (get_u64(cmp + 64 + 8 * t) != ((2ull << 62) | excl)) return ORC_ERR_FORMAT;
        }
    }
    if (excl != pb) return ORC_ERR_FORMAT;
    return ORC_OK;
}

int oracle_decompress(const uint8_t *cmp, uint64_t cmp_bytes, void *out, uint64_t n,
                      int dtype) {
    if (cmp_bytes < 64 || cmp[5] != (uint8_t)dtype) return ORC_ERR_FORMAT;
    int32_t *q = (int32_t *)malloc((size_t)(n ? n : 1) * sizeof(int32_t));
    if (!q) return ORC_ERR_ARG;
    int L = 32;
    int rc = decode_stream(cmp, cmp_bytes, n, q, &L);
    if (rc == ORC_OK) oracle_dequantize(q, n, dtype, get_f64(cmp + 32), out);
    free(q);
    return rc;
}

int oracle_decompress_ints(const uint8_t *cmp, uint64_t cmp_bytes, int32_t *q, uint64_t n) {
    int L = 32;
    return decode_stream(cmp, cmp_bytes, n, q, &L);
}

/* ---------- NEXT #3: multi-dimensional Lorenzo (Table VI; FORMAT.md §7) ---------- */

typedef struct {
    uint64_t nx, ny, nz;  /* field extents, x fastest */
    int ndim, bx, by, bz; /* block shape: 8x8 (2D) or 4x4x4 (3D), 64 values */
    uint64_t nbx, nby, nbz, nb;
} ndgeom_t;

static int nd_setup(ndgeom_t *g, uint64_t nx, uint64_t ny, uint64_t nz, int ndim) {
    if (ndim != 2 && ndim != 3) return ORC_ERR_ARG;
    if (ndim == 2) nz = 1;
    g->nx = nx;
    g->ny = ny;
    g->nz = nz;
    g->ndim = ndim;
    g->bx = g->by = (ndim == 2) ? 8 : 4;
    g->bz = (ndim == 2) ? 1 : 4;
    g->nbx = (nx + g->bx - 1) / g->bx;
    g->nby = (ny + g->by - 1) / g->by;
    g->nbz = (nz + g->bz - 1) / g->bz;
    g->nb = g->nbx * g->nby * g->nbz;
    return ORC_OK;
}

/* field linear index of value i (x fastest inside the block) of block b (blocks in
 * x-fastest order over the block grid), or -1 outside the field */
static int64_t nd_index(const ndgeom_t *g, uint64_t b, int i) {
    uint64_t cbx = b % g->nbx, cby = (b / g->nbx) % g->nby, cbz = b / (g->nbx * g->nby);
    int ix = i % g->bx, iy = (i / g->bx) % g->by, iz = i / (g->bx * g->by);
    uint64_t x = cbx * g->bx + ix, y = cby * g->by + iy, z = cbz * g->bz + iz;
    if (x >= g->nx || y >= g->ny || z >= g->nz) return -1;
    return (int64_t)((z * g->ny + y) * g->nx + x);
}

/* q at in-block (ix, iy, iz); 0 outside the block (block-local prediction, like q_-1) */
static int64_t qat(const int32_t *q, const ndgeom_t *g, int ix, int iy, int iz) {
    if (ix < 0 || iy < 0 || iz < 0) return 0;
    return q[(iz * g->by + iy) * g->bx + ix];
}

/* Lorenzo prediction of value (ix, iy, iz) from its 3 (2D) / 7 (3D) lower neighbours
 * ("2D and 3D processing involve calculations with 3 and 7 adjacent data points") */
static int64_t lorenzo_pred(const int32_t *q, const ndgeom_t *g, int ix, int iy, int iz) {
    if (g->ndim == 2)
        return qat(q, g, ix - 1, iy, 0) + qat(q, g, ix, iy - 1, 0) - qat(q, g, ix - 1, iy - 1, 0);
    return qat(q, g, ix - 1, iy, iz) + qat(q, g, ix, iy - 1, iz) + qat(q, g, ix, iy, iz - 1) -
           qat(q, g, ix - 1, iy - 1, iz) - qat(q, g, ix - 1, iy, iz - 1) -
           qat(q, g, ix, iy - 1, iz - 1) + qat(q, g, ix - 1, iy - 1, iz - 1);
}

uint64_t oracle_compress_bound_nd(uint64_t nx, uint64_t ny, uint64_t nz, int ndim) {
    ndgeom_t g;
    if (nd_setup(&g, nx, ny, nz, ndim)) return 0;
    uint64_t T = (g.nb + BPT - 1) / BPT;
    uint64_t O = roundup16(64 + 8 * T), D = roundup16(O + g.nb);
    return roundup16(D + 4 * 64 * g.nb);
}

int oracle_compress_nd(const void *x, uint64_t nx, uint64_t ny, uint64_t nz, int ndim,
                       int dtype, double eb, int eb_mode, int enc_mode, uint8_t *out,
                       uint64_t *out_bytes) {
    ndgeom_t g;
    if (nd_setup(&g, nx, ny, nz, ndim) || (dtype != ORC_F32 && dtype != ORC_F64) ||
        (enc_mode != ORC_PLAIN && enc_mode != ORC_OUTLIER) || nx >= (1ull << 32) ||
        ny >= (1ull << 32))
        return ORC_ERR_ARG;
    uint64_t n = g.nx * g.ny * g.nz;
    if (!x && n) return ORC_ERR_ARG;
    double eb_abs = 0.0;
    int rc = oracle_resolve_eb(x, n, dtype, eb, eb_mode, &eb_abs);
    if (rc != ORC_OK) return rc;
    int32_t *q = (int32_t *)malloc((size_t)(n ? n : 1) * sizeof(int32_t));
    if (!q) return ORC_ERR_ARG;
    /* ❶ with the tighter range of this predictor (|d| <= 2^ndim * max|q|) */
    int status = quantize_p(x, n, dtype, eb_abs, q, ndim - 1);

    uint64_t T = (g.nb + BPT - 1) / BPT;
    uint64_t O = roundup16(64 + 8 * T), D = roundup16(O + g.nb);
    uint64_t excl = 0, total;
    if (status == ORC_OK) {
        memset(out, 0, (size_t)D);
        int32_t blk[64], d[64];
        int valid[64];
        uint8_t buf[4 * 64 + 8];
        for (uint64_t b = 0; b < g.nb; b++) {
            for (int i = 0; i < 64; i++) {
                int64_t idx = nd_index(&g, b, i);
                valid[i] = idx >= 0;
                blk[i] = valid[i] ? q[idx] : 0;
            }
            /* residuals: value minus its Lorenzo prediction; 0 outside the field */
            for (int i = 0; i < 64; i++) {
                int ix = i % g.bx, iy = (i / g.bx) % g.by, iz = i / (g.bx * g.by);
                d[i] = valid[i] ? (int32_t)(blk[i] - lorenzo_pred(blk, &g, ix, iy, iz)) : 0;
            }
            uint8_t ob_byte = 0;
            int size = fle_encode(d, 64, enc_mode, &ob_byte, buf);
            out[O + b] = ob_byte;
            memcpy(out + D + excl, buf, (size_t)size);
            excl += (uint64_t)size;
            if ((b + 1) % BPT == 0 || b + 1 == g.nb) put_u64(out + 64 + 8 * (b / BPT), (2ull << 62) | excl);
        }
        total = roundup16(D + excl);
        memset(out + D + excl, 0, (size_t)(total - D - excl));
    } else {
        excl = 0;
        total = roundup16(D);
        memset(out, 0, (size_t)total);
    }
    free(q);
    write_header(out, dtype, enc_mode, 64, eb_mode, status, n, eb, eb_abs, excl, total);
    out[12] = (uint8_t)(ndim - 1);
    put_u32(out + 56, (uint32_t)g.nx);
    put_u32(out + 60, (uint32_t)g.ny);
    *out_bytes = total;
    return status;
}

int oracle_decompress_nd(const uint8_t *cmp, uint64_t cmp_bytes, void *out, uint64_t nx,
                         uint64_t ny, uint64_t nz, int ndim, int dtype) {
    ndgeom_t g;
    if (nd_setup(&g, nx, ny, nz, ndim)) return ORC_ERR_ARG;
    uint64_t n = g.nx * g.ny * g.nz;
    if (cmp_bytes < 64 || get_u32(cmp) != MAGIC || cmp[4] != 1 || cmp[5] != (uint8_t)dtype ||
        cmp[7] != 6 || cmp[12] != (uint8_t)(ndim - 1) || get_u16(cmp + 10) != BPT ||
        get_u64(cmp + 16) != n || get_u32(cmp + 56) != (uint32_t)g.nx ||
        get_u32(cmp + 60) != (uint32_t)g.ny)
        return ORC_ERR_FORMAT;
    if (cmp[9] == ORC_ERR_RANGE) return ORC_ERR_RANGE;
    if (cmp[9] != 0) return ORC_ERR_FORMAT;
    uint64_t T = (g.nb + BPT - 1) / BPT;
    uint64_t O = roundup16(64 + 8 * T), D = roundup16(O + g.nb);
    uint64_t pb = get_u64(cmp + 40), total = get_u64(cmp + 48);
    if (total != roundup16(D + pb) || total > cmp_bytes) return ORC_ERR_FORMAT;
    int32_t *q = (int32_t *)malloc((size_t)(n ? n : 1) * sizeof(int32_t));
    if (!q) return ORC_ERR_ARG;
    uint64_t excl = 0;
    int32_t d[64], blk[64];
    int rc = ORC_OK;
    for (uint64_t b = 0; b < g.nb && rc == ORC_OK; b++) {
        int size = oracle_block_size(cmp[O + b], 64);
        if (size < 0 || excl + (uint64_t)size > pb) {
            rc = ORC_ERR_FORMAT;
            break;
        }
        fle_decode(cmp[O + b], cmp + D + excl, 64, d);
        excl += (uint64_t)size;
        /* inverse Lorenzo in index order: value = residual + prediction */
        for (int i = 0; i < 64; i++) {
            int ix = i % g.bx, iy = (i / g.bx) % g.by, iz = i / (g.bx * g.by);
            blk[i] = (int32_t)((int64_t)d[i] + lorenzo_pred(blk, &g, ix, iy, iz));
        }
        for (int i = 0; i < 64; i++) {
            int64_t idx = nd_index(&g, b, i);
            if (idx >= 0) q[idx] = blk[i];
        }
        if (((b + 1) % BPT == 0 || b + 1 == g.nb) &&
            get_u64(cmp + 64 + 8 * (b / BPT)) != ((2ull << 62) | excl))
            rc = ORC_ERR_FORMAT;
    }
    if (rc == ORC_OK && excl != pb) rc = ORC_ERR_FORMAT;
    if (rc == ORC_OK) oracle_dequantize(q, n, dtype, get_f64(cmp + 32), out);
    free(q);
    return rc;
}
