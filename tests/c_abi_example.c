/*
 * c_abi_example.c -- the C ABI used from plain C (no Python, no PyTorch): screen a population
 * read from a binary file and write the conjunctions to another (tests/test_gpu_c_abi.py compiles
 * and runs it and compares the output with the Python binding's result).
 *
 *   gcc -std=c11 -O2 -I include tests/c_abi_example.c -L<pkg> -lcdscreen -o c_abi_example
 *   ./c_abi_example pop.f64 n t0 t1 dt d mode out.bin
 *
 * pop.f64: six fp64 arrays of n values each, in the cd_elements order (a, e, inc, raan, argp,
 * nu0); out.bin: count (uint64) followed by count cd_conjunction records.  mode: 0 grid, 1 hybrid.
 */
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>

#include "cdscreen.h"

int main(int argc, char** argv)
{
    if (argc != 9) {
        fprintf(stderr, "usage: %s pop.f64 n t0 t1 dt d mode out.bin\n", argv[0]);
        return 2;
    }
    const size_t n = (size_t)strtoull(argv[2], NULL, 10);
    const double t0 = atof(argv[3]), t1 = atof(argv[4]), dt = atof(argv[5]), d = atof(argv[6]);
    const cd_mode mode = (cd_mode)atoi(argv[7]);
    double* buf = (double*)malloc(sizeof(double) * 6 * (n ? n : 1));
    FILE* f = fopen(argv[1], "rb");
    if (!buf || !f || fread(buf, sizeof(double), 6 * n, f) != 6 * n) {
        fprintf(stderr, "cannot read %s\n", argv[1]);
        return 1;
    }
    fclose(f);
    const cd_elements el = {buf, buf + n, buf + 2 * n, buf + 3 * n, buf + 4 * n, buf + 5 * n};

    cd_options opt;
    cd_options_init(&opt);
    cd_stats st;
    opt.stats = &st;
    cd_conjunctions out;
    const cd_status s = cd_screen_ex(&el, n, t0, t1, dt, d, mode, &opt, &out);
    if (s != CD_OK) {
        fprintf(stderr, "cd_screen_ex: %s: %s\n", cd_status_str(s), cd_last_error());
        return 1;
    }
    /* an invalid call reports CD_EINVAL with a message and an empty result */
    cd_conjunctions bad;
    if (cd_screen(&el, n, t1, t0, dt, d, mode, &bad) != CD_EINVAL || bad.count != 0 || bad.data) {
        fprintf(stderr, "t1 < t0 was not rejected\n");
        return 1;
    }
    FILE* o = fopen(argv[8], "wb");
    const uint64_t cnt = out.count;
    if (!o || fwrite(&cnt, sizeof cnt, 1, o) != 1 ||
        (cnt && fwrite(out.data, sizeof(cd_conjunction), cnt, o) != cnt)) {
        fprintf(stderr, "cannot write %s\n", argv[8]);
        return 1;
    }
    fclose(o);
    printf("abi %d: %llu conjunctions, %llu candidates, %llu steps, %llu kernel launches, %.3f ms\n",
           cd_abi_version(), (unsigned long long)cnt, (unsigned long long)st.candidates,
           (unsigned long long)st.steps, (unsigned long long)st.kernel_launches, st.ms_total);
    cd_conjunctions_free(&out);
    cd_release_caches(-1);
    free(buf);
    return 0;
}
