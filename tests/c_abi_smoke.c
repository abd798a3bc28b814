/* c_abi_smoke.c -- librap.so used from plain C (no torch, no Python): the boundary really is a
 * C ABI.  Transposes a 300 x 257 float matrix (ragged tails) under every layout and checks
 * dst[c][r] == src[r][c] bit for bit; runs a 100000-trial w=32 sweep and checks the invariants
 * Theorem 2 fixes (RAP contiguous and stride congestion 1 on every trial) and the
 * RAW stride congestion w.  Exit code 0 = pass.
 * Build: gcc -O2 -std=c99 -D_GNU_SOURCE -I include tests/c_abi_smoke.c -o c_abi_smoke -ldl
 * Run:   ./c_abi_smoke paper_conf_icppw_nakanomi14_b200/librap.so libcudart.so.12
 * (librap.so and the CUDA runtime are dlopen'ed, so the program builds without a GPU). */
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>
#include <dlfcn.h>

#include "rap.h"

/* the CUDA runtime entry points this program needs, resolved at run time */
typedef int (*malloc_fn)(void **, size_t);
typedef int (*free_fn)(void *);
typedef int (*memcpy_fn)(void *, const void *, size_t, int);
typedef int (*sync_fn)(void);

int main(int argc, char **argv) {
    if (argc < 3) { fprintf(stderr, "usage: %s librap.so libcudart.so\n", argv[0]); return 2; }
    void *rap = dlopen(argv[1], RTLD_NOW), *rt = dlopen(argv[2], RTLD_NOW);
    if (!rap || !rt) { fprintf(stderr, "dlopen: %s\n", dlerror()); return 2; }
    malloc_fn cmalloc = (malloc_fn)dlsym(rt, "cudaMalloc");
    free_fn cfree = (free_fn)dlsym(rt, "cudaFree");
    memcpy_fn cmemcpy = (memcpy_fn)dlsym(rt, "cudaMemcpy");
    sync_fn csync = (sync_fn)dlsym(rt, "cudaDeviceSynchronize");
    int (*abi)(void) = (int (*)(void))dlsym(rap, "rap_abi_version");
    rap_status_t (*tr)(const void *, void *, int64_t, int64_t, int64_t, int64_t, uint32_t, rap_layout_t, uint64_t,
                       void *) = dlsym(rap, "rap_transpose");
    rap_status_t (*sw)(uint32_t, uint32_t, uint32_t, uint64_t, uint64_t, uint64_t, uint64_t *, void *) =
        dlsym(rap, "rap_congestion_sweep");
    const char *(*str)(rap_status_t) = dlsym(rap, "rap_status_str");
    if (!cmalloc || !cfree || !cmemcpy || !csync || !abi || !tr || !sw || !str) { fprintf(stderr, "dlsym\n"); return 2; }
    if (abi() != RAP_ABI_VERSION) { fprintf(stderr, "abi %d\n", abi()); return 1; }

    const int64_t R = 300, C = 257;
    uint32_t *h = malloc(R * C * 4), *ht = malloc(R * C * 4);
    for (int64_t i = 0; i < R * C; ++i) h[i] = (uint32_t)(i * 2654435761u) ^ 0x7fc00001u;
    void *d = NULL, *dt = NULL;
    if (cmalloc(&d, R * C * 4) || cmalloc(&dt, R * C * 4)) return 2;
    cmemcpy(d, h, R * C * 4, 1 /* H2D */);
    for (int lay = RAP_LAYOUT_RAW; lay <= RAP_LAYOUT_RAP; ++lay) {
        memset(ht, 0, R * C * 4);
        rap_status_t s = tr(d, dt, R, C, C, R, 4, (rap_layout_t)lay, 42, NULL);
        if (s != RAP_OK) { fprintf(stderr, "transpose: %s\n", str(s)); return 1; }
        csync();
        cmemcpy(ht, dt, R * C * 4, 2 /* D2H */);
        for (int64_t r = 0; r < R; ++r)
            for (int64_t c = 0; c < C; ++c)
                if (ht[c * R + r] != h[r * C + c]) { fprintf(stderr, "layout %d mismatch at %ld,%ld\n", lay, (long)r, (long)c); return 1; }
    }
    /* argument errors come back before anything is launched */
    if (tr(d, d, R, C, C, R, 4, RAP_LAYOUT_RAP, 0, NULL) != RAP_ERR_ALIAS) return 1;
    if (tr(d, dt, R, C, C, R, 3, RAP_LAYOUT_RAP, 0, NULL) != RAP_ERR_INVALID_ARG) return 1;

    uint64_t *dh = NULL, hh[5 * 3 * 33];
    if (cmalloc((void **)&dh, sizeof(hh))) return 2;
    memset(hh, 0, sizeof(hh));
    cmemcpy(dh, hh, sizeof(hh), 1);
    const uint64_t N = 100000;
    rap_status_t s = sw(32, 31, 7, 1, 0, N, dh, NULL);
    if (s != RAP_OK) { fprintf(stderr, "sweep: %s\n", str(s)); return 1; }
    csync();
    cmemcpy(hh, dh, sizeof(hh), 2);
    /* [pattern][scheme][c]: contiguous row, stride row (patterns 0, 1); schemes RAW, RAS, RAP */
    for (int sc = 0; sc < 3; ++sc)
        if (hh[(0 * 3 + sc) * 33 + 1] != N) { fprintf(stderr, "contiguous scheme %d\n", sc); return 1; }
    if (hh[(1 * 3 + 2) * 33 + 1] != N) { fprintf(stderr, "RAP stride\n"); return 1; }
    if (hh[(1 * 3 + 0) * 33 + 32] != N) { fprintf(stderr, "RAW stride\n"); return 1; }
    cfree(d); cfree(dt); cfree(dh); free(h); free(ht);
    printf("c_abi_smoke ok\n");
    return 0;
}
