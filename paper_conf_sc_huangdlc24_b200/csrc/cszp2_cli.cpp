// cszp2 — command-line front end over the C ABI (SURVEY §8(b) "CLI", mirroring the
// paper's artifact binaries): read a raw f32/f64 field from a file, compress
// and decompress it on the GPU, report end-to-end device throughput (Fig 3:
// events around the API call, device buffer to device buffer), compression ratio, PSNR,
// and check the error bound on every value.
//
//   cszp2 -m P|O (-a|-r) file.{f32,f64} eb [-t f32|f64] [-n count] [-z out.cszp]
//         [-d out.{f32,f64}] [-w warmups] [-k reps]
//   cszp2 -x in.cszp n (-t f32|f64) out.{f32,f64}      decompress a stored stream
//
// Everything goes through libcszp2.so's extern "C" entry points (include/cszp2.h);
// this file only moves bytes between files, host and device and does the reporting.
#include <cuda_runtime.h>

#include <cmath>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <string>
#include <vector>

#include "cszp2.h"

namespace {

void usage(FILE *f) {
    std::fprintf(f,
                 "usage: cszp2 -m P|O (-a|-r) file.{f32,f64} eb [-t f32|f64] [-n count]\n"
                 "             [-z out.cszp] [-d out.{f32,f64}] [-w warmups] [-k reps]\n"
                 "       cszp2 -x in.cszp n -t f32|f64 out.{f32,f64}\n"
                 "  -m P|O   Plain-FLE or Outlier-FLE (CUSZP2-P / CUSZP2-O)\n"
                 "  -a | -r  eb is absolute, or relative to the value range (REL)\n"
                 "  -t       element type (default: from the file extension, else f32)\n"
                 "  -n       number of values (default: file size / element size)\n"
                 "  -z / -d  also write the compressed stream / the reconstruction\n"
                 "  -w / -k  untimed warm-up runs (default 2) / timed runs (default 5)\n"
                 "prints compression and decompression end-to-end GB/s (device buffer to\n"
                 "device buffer, CUDA events around the API call), compression ratio,\n"
                 "PSNR and the result of the error-bound check on every value.\n");
}

#define CK(call)                                                                        \
    do {                                                                                \
        cudaError_t e_ = (call);                                                        \
        if (e_ != cudaSuccess) {                                                        \
            std::fprintf(stderr, "cszp2: %s: %s\n", #call, cudaGetErrorString(e_));     \
            return 2;                                                                   \
        }                                                                               \
    } while (0)
#define CZ(call)                                                                        \
    do {                                                                                \
        int r_ = (call);                                                                \
        if (r_ != CSZP2_OK) {                                                           \
            std::fprintf(stderr, "cszp2: %s returned %d\n", #call, r_);                 \
            return 2;                                                                   \
        }                                                                               \
    } while (0)

bool read_file(const char *path, std::vector<uint8_t> &buf) {
    FILE *f = std::fopen(path, "rb");
    if (!f) return false;
    std::fseek(f, 0, SEEK_END);
    long sz = std::ftell(f);
    std::fseek(f, 0, SEEK_SET);
    buf.resize(sz > 0 ? static_cast<size_t>(sz) : 0);
    bool ok = buf.empty() || std::fread(buf.data(), 1, buf.size(), f) == buf.size();
    std::fclose(f);
    return ok;
}

bool write_file(const char *path, const void *p, size_t n) {
    FILE *f = std::fopen(path, "wb");
    if (!f) return false;
    bool ok = n == 0 || std::fwrite(p, 1, n, f) == n;
    return std::fclose(f) == 0 && ok;
}

int dtype_from_name(const char *s) {
    if (!std::strcmp(s, "f32")) return CSZP2_F32;
    if (!std::strcmp(s, "f64")) return CSZP2_F64;
    return -1;
}

int dtype_from_path(const std::string &p) {
    auto ends = [&](const char *e) {
        size_t n = std::strlen(e);
        return p.size() >= n && p.compare(p.size() - n, n, e) == 0;
    };
    if (ends(".f64") || ends(".d64")) return CSZP2_F64;
    return CSZP2_F32;
}

template <typename T>
void stats(const T *x, const T *y, uint64_t n, double eb_abs, double *psnr, uint64_t *bad,
           double *max_err) {
    // error bound as in tests (R-10): x' is rounded to T
    const double rel = sizeof(T) == 4 ? std::ldexp(1.0, -21) : std::ldexp(1.0, -50);
    const double slack = sizeof(T) == 4 ? std::ldexp(1.0, -20) : std::ldexp(1.0, -40);
    double mn = INFINITY, mx = -INFINITY, se = 0.0, me = 0.0;
    uint64_t b = 0;
    for (uint64_t i = 0; i < n; i++) {
        const double a = static_cast<double>(x[i]), c = static_cast<double>(y[i]);
        if (a < mn) mn = a;
        if (a > mx) mx = a;
        const double e = std::fabs(a - c);
        se += e * e;
        if (e > me) me = e;
        if (!(e <= eb_abs * (1.0 + slack) + rel * std::fmax(std::fabs(a), std::fabs(c)))) b++;
    }
    const double mse = n ? se / static_cast<double>(n) : 0.0;
    *psnr = mse > 0 ? 20.0 * std::log10(mx - mn) - 10.0 * std::log10(mse) : INFINITY;
    *bad = b;
    *max_err = me;
}

int decompress_file(int argc, char **argv) {
    // cszp2 -x in.cszp n -t f32|f64 out
    if (argc != 7 || std::strcmp(argv[4], "-t")) {
        usage(stderr);
        return 1;
    }
    const uint64_t n = std::strtoull(argv[3], nullptr, 10);
    const int dt = dtype_from_name(argv[5]);
    if (dt < 0) {
        usage(stderr);
        return 1;
    }
    std::vector<uint8_t> cmp;
    if (!read_file(argv[2], cmp)) {
        std::fprintf(stderr, "cszp2: cannot read %s\n", argv[2]);
        return 1;
    }
    const size_t w = dt == CSZP2_F32 ? 4 : 8;
    void *d_cmp = nullptr, *d_out = nullptr;
    int *d_st = nullptr;
    CK(cudaMalloc(&d_cmp, cmp.size() + 16));
    CK(cudaMalloc(&d_out, n * w + 16));
    CK(cudaMalloc(&d_st, sizeof(int)));
    CK(cudaMemset(d_st, 0, sizeof(int)));
    CK(cudaMemcpy(d_cmp, cmp.data(), cmp.size(), cudaMemcpyHostToDevice));
    CZ(cszp2_decompress(d_cmp, d_out, n, dt, d_st, nullptr));
    int st = 0;
    CK(cudaMemcpy(&st, d_st, sizeof(int), cudaMemcpyDeviceToHost));
    if (st != CSZP2_OK) {
        std::fprintf(stderr, "cszp2: stream status %d (%s)\n", st, st == CSZP2_ERR_RANGE ? "RANGE" : "FORMAT");
        return 2;
    }
    std::vector<uint8_t> y(n * w);
    CK(cudaMemcpy(y.data(), d_out, n * w, cudaMemcpyDeviceToHost));
    if (!write_file(argv[6], y.data(), y.size())) {
        std::fprintf(stderr, "cszp2: cannot write %s\n", argv[6]);
        return 1;
    }
    std::printf("decompressed %llu values to %s\n", static_cast<unsigned long long>(n), argv[6]);
    cudaFree(d_cmp);
    cudaFree(d_out);
    cudaFree(d_st);
    return 0;
}

}  // namespace

int main(int argc, char **argv) {
    if (argc < 2 || !std::strcmp(argv[1], "-h") || !std::strcmp(argv[1], "--help")) {
        usage(argc < 2 ? stderr : stdout);
        return argc < 2 ? 1 : 0;
    }
    if (!std::strcmp(argv[1], "-x")) return decompress_file(argc, argv);

    int enc = -1, ebm = -1, dt = -1, warm = 2, reps = 5;
    const char *path = nullptr, *zpath = nullptr, *dpath = nullptr;
    double eb = 0.0;
    bool have_eb = false;
    uint64_t n_arg = 0;
    for (int i = 1; i < argc; i++) {
        const char *a = argv[i];
        auto next = [&]() -> const char * { return i + 1 < argc ? argv[++i] : nullptr; };
        if (!std::strcmp(a, "-m")) {
            const char *v = next();
            if (!v) break;
            enc = (v[0] == 'P' || v[0] == 'p') ? CSZP2_ENC_PLAIN : (v[0] == 'O' || v[0] == 'o') ? CSZP2_ENC_OUTLIER : -2;
        } else if (!std::strcmp(a, "-a")) {
            ebm = CSZP2_EB_ABS;
        } else if (!std::strcmp(a, "-r")) {
            ebm = CSZP2_EB_REL;
        } else if (!std::strcmp(a, "-t")) {
            const char *v = next();
            dt = v ? dtype_from_name(v) : -2;
            if (dt < 0) dt = -2;
        } else if (!std::strcmp(a, "-n")) {
            const char *v = next();
            n_arg = v ? std::strtoull(v, nullptr, 10) : 0;
        } else if (!std::strcmp(a, "-z")) {
            zpath = next();
        } else if (!std::strcmp(a, "-d")) {
            dpath = next();
        } else if (!std::strcmp(a, "-w")) {
            const char *v = next();
            warm = v ? std::atoi(v) : -1;
        } else if (!std::strcmp(a, "-k")) {
            const char *v = next();
            reps = v ? std::atoi(v) : 0;
        } else if (!path) {
            path = a;
        } else if (!have_eb) {
            char *end = nullptr;
            eb = std::strtod(a, &end);
            have_eb = end && *end == '\0';
        } else {
            usage(stderr);
            return 1;
        }
    }
    if (enc < 0 || ebm < 0 || dt == -2 || !path || !have_eb || !(eb > 0.0) || warm < 0 || reps < 1) {
        usage(stderr);
        return 1;
    }
    if (dt < 0) dt = dtype_from_path(path);
    const size_t w = dt == CSZP2_F32 ? 4 : 8;

    std::vector<uint8_t> host;
    if (!read_file(path, host)) {
        std::fprintf(stderr, "cszp2: cannot read %s\n", path);
        return 1;
    }
    const uint64_t n = n_arg ? n_arg : host.size() / w;
    if (n * w > host.size()) {
        std::fprintf(stderr, "cszp2: %s holds fewer than %llu values\n", path, static_cast<unsigned long long>(n));
        return 1;
    }

    const uint64_t bound = cszp2_compress_bound(n, dt);
    void *d_in = nullptr, *d_cmp = nullptr, *d_out = nullptr;
    uint64_t *d_bytes = nullptr;
    int *d_st = nullptr;
    CK(cudaMalloc(&d_in, n * w + 16));
    CK(cudaMalloc(&d_cmp, bound));
    CK(cudaMalloc(&d_out, n * w + 16));
    CK(cudaMalloc(&d_bytes, sizeof(uint64_t)));
    CK(cudaMalloc(&d_st, sizeof(int)));
    CK(cudaMemset(d_st, 0, sizeof(int)));
    CK(cudaMemcpy(d_in, host.data(), n * w, cudaMemcpyHostToDevice));
    cudaStream_t st;
    CK(cudaStreamCreate(&st));
    cudaEvent_t e0, e1, e2;
    CK(cudaEventCreate(&e0));
    CK(cudaEventCreate(&e1));
    CK(cudaEventCreate(&e2));

    for (int i = 0; i < warm; i++) {
        CZ(cszp2_compress(d_in, n, dt, eb, ebm, enc, d_cmp, d_bytes, st));
        CZ(cszp2_decompress(d_cmp, d_out, n, dt, d_st, st));
    }
    float tc = 0.f, td = 0.f;
    for (int i = 0; i < reps; i++) {
        CK(cudaEventRecord(e0, st));
        CZ(cszp2_compress(d_in, n, dt, eb, ebm, enc, d_cmp, d_bytes, st));
        CK(cudaEventRecord(e1, st));
        CZ(cszp2_decompress(d_cmp, d_out, n, dt, d_st, st));
        CK(cudaEventRecord(e2, st));
        CK(cudaEventSynchronize(e2));
        float a = 0.f, b = 0.f;
        CK(cudaEventElapsedTime(&a, e0, e1));
        CK(cudaEventElapsedTime(&b, e1, e2));
        tc += a;
        td += b;
    }
    tc /= reps;
    td /= reps;

    uint64_t bytes = 0;
    int status = 0;
    CK(cudaMemcpy(&bytes, d_bytes, sizeof(bytes), cudaMemcpyDeviceToHost));
    CK(cudaMemcpy(&status, d_st, sizeof(int), cudaMemcpyDeviceToHost));
    cszp2_header hdr;
    CZ(cszp2_read_header(d_cmp, &hdr, st));
    const double gb = static_cast<double>(n * w) / 1e9;
    std::printf("cuSZp2 (B200, %s, %s-FLE, %s %g) finished on %llu values\n", dt == CSZP2_F32 ? "f32" : "f64",
                enc == CSZP2_ENC_PLAIN ? "Plain" : "Outlier", ebm == CSZP2_EB_REL ? "REL" : "ABS", eb,
                static_cast<unsigned long long>(n));
    std::printf("compression   end-to-end speed: %f GB/s\n", tc > 0 ? gb / (tc * 1e-3) : 0.0);
    std::printf("decompression end-to-end speed: %f GB/s\n", td > 0 ? gb / (td * 1e-3) : 0.0);
    std::printf("compression ratio: %f\n", bytes ? static_cast<double>(n * w) / static_cast<double>(bytes) : 0.0);
    if (status != CSZP2_OK) {
        std::printf("stream status: %s\nFail error check!\n", status == CSZP2_ERR_RANGE ? "RANGE" : "FORMAT");
        return 3;
    }
    std::vector<uint8_t> y(n * w);
    CK(cudaMemcpy(y.data(), d_out, n * w, cudaMemcpyDeviceToHost));
    double psnr = 0.0, max_err = 0.0;
    uint64_t bad = 0;
    if (dt == CSZP2_F32)
        stats(reinterpret_cast<const float *>(host.data()), reinterpret_cast<const float *>(y.data()), n,
              hdr.eb_abs, &psnr, &bad, &max_err);
    else
        stats(reinterpret_cast<const double *>(host.data()), reinterpret_cast<const double *>(y.data()), n,
              hdr.eb_abs, &psnr, &bad, &max_err);
    std::printf("PSNR: %f dB\n", psnr);
    std::printf("eb_abs: %.17g, max |x - x'|: %.17g\n", hdr.eb_abs, max_err);
    if (zpath) {
        std::vector<uint8_t> z(bytes);
        CK(cudaMemcpy(z.data(), d_cmp, bytes, cudaMemcpyDeviceToHost));
        if (!write_file(zpath, z.data(), z.size())) std::fprintf(stderr, "cszp2: cannot write %s\n", zpath);
    }
    if (dpath && !write_file(dpath, y.data(), y.size())) std::fprintf(stderr, "cszp2: cannot write %s\n", dpath);
    if (bad) {
        std::printf("Fail error check! (%llu values exceed the bound)\n", static_cast<unsigned long long>(bad));
        return 3;
    }
    std::printf("Pass error check!\n");
    cudaFree(d_in);
    cudaFree(d_cmp);
    cudaFree(d_out);
    cudaFree(d_bytes);
    cudaFree(d_st);
    cudaStreamDestroy(st);
    return 0;
}
