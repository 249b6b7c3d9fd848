/* harris_c.c -- the C-ABI used from plain C (no Python, no torch): builds the
 * paper's Harris DAG (Fig. 3), plans it with Alg. 1 under the
 * paper's and the B200 profile, prints the plans, and -- given "run" and a GPU
 * -- runs the fused plan on a synthetic image through kf_run and kf_run_host.
 *
 *   gcc -std=c99 -Wall -I include examples/harris_c.c -L paper_conf_cgo_qiaorht19_b200 \
 *       -lkfuse -Wl,-rpath,$PWD/paper_conf_cgo_qiaorht19_b200 -o harris_c && ./harris_c [run]
 */
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include "kfuse.h"

#define CHECK(x)                                                                   \
    do {                                                                           \
        kf_status s_ = (x);                                                        \
        if (s_ != KF_OK) {                                                         \
            fprintf(stderr, "%s failed: %d %s\n", #x, (int)s_, kf_last_error());   \
            return 1;                                                              \
        }                                                                          \
    } while (0)

static int local3(kf_pipeline *p, int in, const double *m, int32_t *out)
{
    return (int)kf_add_local_op(p, in, m, 3, 3, KF_CLAMP, 0.0, NULL, 0, NULL, out);
}

int main(int argc, char **argv)
{
    const int W = 512, H = 384;
    const double sobel_x[9] = {-1, 0, 1, -2, 0, 2, -1, 0, 1};
    const double sobel_y[9] = {-1, -2, -1, 0, 0, 0, 1, 2, 1};
    const double gauss[9] = {1 / 16., 2 / 16., 1 / 16., 2 / 16., 4 / 16., 2 / 16., 1 / 16., 2 / 16., 1 / 16.};
    const kf_instr sq[3] = {{KF_OP_LOAD, 0, 0}, {KF_OP_LOAD, 0, 0}, {KF_OP_MUL, 0, 0}};
    const kf_instr prod[3] = {{KF_OP_LOAD, 0, 0}, {KF_OP_LOAD, 1, 0}, {KF_OP_MUL, 0, 0}};
    /* R = gx*gy - gxy^2 - k (gx+gy)^2 */
    const kf_instr resp[17] = {{KF_OP_LOAD, 0, 0}, {KF_OP_LOAD, 1, 0}, {KF_OP_MUL, 0, 0}, {KF_OP_LOAD, 2, 0},
                               {KF_OP_LOAD, 2, 0}, {KF_OP_MUL, 0, 0},  {KF_OP_SUB, 0, 0}, {KF_OP_CONST, 0, 0.04},
                               {KF_OP_LOAD, 0, 0}, {KF_OP_LOAD, 1, 0}, {KF_OP_ADD, 0, 0}, {KF_OP_MUL, 0, 0},
                               {KF_OP_LOAD, 0, 0}, {KF_OP_LOAD, 1, 0}, {KF_OP_ADD, 0, 0}, {KF_OP_MUL, 0, 0},
                               {KF_OP_SUB, 0, 0}};
    const kf_cost two = {2, 0};
    kf_pipeline *p;
    int32_t in, dx, dy, sx, sy, sxy, gx, gy, gxy, hc;
    CHECK(kf_pipeline_create(W, H, KF_F32, &p));
    CHECK(kf_add_input(p, &in));
    CHECK((kf_status)local3(p, in, sobel_x, &dx));
    CHECK((kf_status)local3(p, in, sobel_y, &dy));
    CHECK(kf_add_point_op(p, &dx, 1, sq, 3, &two, NULL, 0, &sx));
    CHECK(kf_add_point_op(p, &dy, 1, sq, 3, &two, NULL, 0, &sy));
    {
        const int32_t ins[2] = {dx, dy};
        CHECK(kf_add_point_op(p, ins, 2, prod, 3, &two, NULL, 0, &sxy));
    }
    CHECK((kf_status)local3(p, sx, gauss, &gx));
    CHECK((kf_status)local3(p, sy, gauss, &gy));
    CHECK((kf_status)local3(p, sxy, gauss, &gxy));
    {
        const int32_t ins[3] = {gx, gy, gxy};
        CHECK(kf_add_point_op(p, ins, 3, resp, 17, NULL, NULL, 0, &hc));
    }
    CHECK(kf_mark_output(p, hc));

    kf_model_params paper, b200;
    kf_model_params_paper(&paper);
    kf_model_params_b200(&b200);
    kf_plan *pp, *pb;
    CHECK(kf_plan_fusion(p, &paper, &pp));
    CHECK(kf_plan_fusion(p, &b200, &pb));
    int64_t q, e;
    CHECK(kf_plan_objective(pp, &q, &e));
    printf("paper profile: %d blocks, beta = %.1f + %lld eps\n", (int)kf_plan_num_blocks(pp), (double)q / (1 << 20),
           (long long)e);
    CHECK(kf_plan_objective(pb, &q, &e));
    printf("b200 profile: %d block(s), %d launch(es), halo rows %d\n", (int)kf_plan_num_blocks(pb),
           (int)kf_plan_num_launches(pb), (int)kf_plan_halo_rows(pb));

    int rc = 0;
    if (argc > 1 && !strcmp(argv[1], "compile")) CHECK(kf_compile_plan(p, pb));   /* NVRTC only, no GPU */
    if (argc > 1 && !strcmp(argv[1], "run")) {
        float *h_in = (float *)malloc(sizeof(float) * W * H), *h_out = (float *)malloc(sizeof(float) * W * H);
        for (int i = 0; i < W * H; i++) h_in[i] = (float)((i * 2654435761u) >> 8 & 0xffff) / 65536.0f;
        const void *hi[1] = {h_in};
        void *ho[1] = {h_out};
        kf_status s = kf_run_host(p, pb, hi, 1, ho, 1, NULL);   /* host buffers: H2D / run / D2H */
        if (s != KF_OK) {
            fprintf(stderr, "kf_run_host: %d %s\n", (int)s, kf_last_error());
            rc = 2;
        } else {
            double sum = 0;
            for (int i = 0; i < W * H; i++) sum += h_out[i];
            printf("ran the fused plan on %dx%d: checksum %.6e\n", W, H, sum);
        }
        free(h_in);
        free(h_out);
    }
    kf_plan_destroy(pp);
    kf_plan_destroy(pb);
    kf_pipeline_destroy(p);
    return rc;
}
