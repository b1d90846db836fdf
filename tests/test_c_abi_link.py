"""The boundary is a plain C ABI: a C99 program that includes only
include/nitro.h links against libnitro.so and calls host-side entry points
(no GPU needed): version, argument errors with their thread-local message,
and the generic code-variant layer's registration of both workloads."""
import os
import subprocess

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

PROG = r"""
#include <stdio.h>
#include <string.h>
#include "nitro.h"
int main(void) {
  nitro_hist *h = NULL;
  nitro_context *ctx = NULL;
  nitro_cv *cv = NULL, *cv2 = NULL;
  if (strstr(nitro_version(), "sm_100a") == NULL) return 10;
  /* samples NULL with n > 0: rejected before any CUDA call */
  if (nitro_hist_create(0, NULL, 10, NULL, 5, 10, &h) != NITRO_E_INVALID_ARG || h != NULL) return 11;
  if (strlen(nitro_last_error()) == 0) return 12;
  if (nitro_hist_create(0, NULL, 0, NULL, 0, 10, &h) != NITRO_E_INVALID_ARG) return 13;   /* nbins 0 */
  if (nitro_context_create(&ctx) != NITRO_OK) return 14;
  if (nitro_cv_create(ctx, "spmv", &cv) != NITRO_OK || nitro_spmv_register(cv) != NITRO_OK) return 15;
  if (nitro_cv_create(ctx, "histogram", &cv2) != NITRO_OK || nitro_hist_register(cv2) != NITRO_OK) return 16;
  if (nitro_hist_register(cv2) != NITRO_E_STATE) return 17;   /* only on a fresh cv */
  nitro_cv_destroy(cv);
  nitro_cv_destroy(cv2);
  nitro_context_destroy(ctx);
  printf("ok\n");
  return 0;
}
"""


def test_plain_c_program_links_and_calls(tmp_path):
    src = tmp_path / "t.c"
    src.write_text(PROG)
    exe = tmp_path / "t"
    libdir = os.path.join(ROOT, "paper_conf_ipps_muralidharanshgc14_b200")
    subprocess.check_call(["gcc", "-std=c99", "-Wall", "-Werror", "-I", os.path.join(ROOT, "include"), str(src),
                           "-L", libdir, "-lnitro", f"-Wl,-rpath,{libdir}", "-o", str(exe)])
    r = subprocess.run([str(exe)], capture_output=True, text=True, timeout=120)
    assert r.returncode == 0 and r.stdout.strip() == "ok", (r.returncode, r.stdout, r.stderr)
