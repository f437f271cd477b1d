/* C99 client of include/checl.h: exercises the handle table without a GPU
 * (run with CHECL_FAKE_DEVICES=2). Prints one line per check; exit 0 = pass. */
#include <stdint.h>
#include <stdio.h>
#include <string.h>

#include "checl.h"

#define CHECK(c)                                          \
  do {                                                    \
    if (!(c)) {                                           \
      fprintf(stderr, "FAIL %s:%d %s\n", __FILE__, __LINE__, #c); \
      return 1;                                           \
    }                                                     \
  } while (0)

int main(void) {
  checl_ctx* ctx = NULL;
  CHECK(checl_version() == 0x00010000u);
  CHECK(checl_create(NULL, &ctx) == CHECL_SUCCESS && ctx);
  checl_handle a = 0, b = 0, z = 0, c = 0;
  CHECK(checl_register_buffer(ctx, 0, (void*)0x100000, 4096, 7, &a) == CHECL_SUCCESS && a == 1);
  CHECK(checl_register_buffer(ctx, 0, (void*)0x101000, 10, 0, &b) == CHECL_SUCCESS && b == 2);
  /* overlap on the same device is rejected, on another device accepted */
  CHECK(checl_register_buffer(ctx, 0, (void*)0x100FFF, 2, 0, &c) == CHECL_ERR_INVALID_VALUE);
  CHECK(checl_register_buffer(ctx, 0, (void*)0x0FFFFF, 2, 0, &c) == CHECL_ERR_INVALID_VALUE);
  CHECK(checl_register_buffer(ctx, 1, (void*)0x100000, 4096, 0, &c) == CHECL_SUCCESS && c == 3);
  /* zero-size buffers: NULL allowed, never overlap */
  CHECK(checl_register_buffer(ctx, 0, NULL, 0, 0, &z) == CHECL_SUCCESS && z == 4);
  CHECK(checl_register_buffer(ctx, 0, NULL, 5, 0, &c) == CHECL_ERR_INVALID_VALUE);
  CHECK(checl_register_buffer(ctx, 9, (void*)0x1, 1, 0, &c) == CHECL_ERR_INVALID_DEVICE);
  CHECK(checl_register_buffer(ctx, 0, (void*)0x1, 1, 0, NULL) == CHECL_ERR_INVALID_VALUE);
  void* p = NULL;
  size_t n = 0;
  int d = -1;
  CHECK(checl_translate(ctx, a, &p, &n, &d) == CHECL_SUCCESS && p == (void*)0x100000 && n == 4096 && d == 0);
  CHECK(checl_translate(ctx, z, &p, &n, &d) == CHECL_SUCCESS && p == NULL && n == 0);
  CHECK(checl_translate(ctx, 0, &p, &n, &d) == CHECL_ERR_INVALID_HANDLE);
  uint64_t nb = 0, tb = 0;
  CHECK(checl_count(ctx, 0, &nb, &tb) == CHECL_SUCCESS && nb == 3 && tb == 4106);
  CHECK(checl_release(ctx, a) == CHECL_SUCCESS);
  CHECK(checl_release(ctx, a) == CHECL_ERR_INVALID_HANDLE);
  CHECK(checl_translate(ctx, a, &p, &n, &d) == CHECL_ERR_INVALID_HANDLE);
  /* released range can be registered again; ids are never reused */
  CHECK(checl_register_buffer(ctx, 0, (void*)0x100000, 4096, 0, &c) == CHECL_SUCCESS && c == 5);
  CHECK(checl_set_staging(ctx, 100, 2) == CHECL_ERR_INVALID_VALUE);
  CHECK(checl_set_staging(ctx, 1 << 20, 9) == CHECL_ERR_INVALID_VALUE);
  CHECK(checl_set_staging(ctx, 1 << 20, 3) == CHECL_SUCCESS);
  CHECK(strcmp(checl_status_string(CHECL_ERR_CRC_MISMATCH), "CHECL_ERR_CRC_MISMATCH") == 0);
  /* wrapped images need no device */
  static uint8_t bytes[4096];
  checl_image* img = NULL;
  const void* v = NULL;
  size_t vn = 0;
  CHECK(checl_image_wrap(bytes, sizeof bytes, &img) == CHECL_SUCCESS);
  CHECK(checl_image_view(img, &v, &vn) == CHECL_SUCCESS && v == bytes && vn == sizeof bytes);
  int loc = -1;
  CHECK(checl_image_info(img, &loc, &d, NULL, NULL) == CHECL_SUCCESS && loc == CHECL_IMAGE_HOST && d == -1);
  /* incremental checkpoint: an unknown dirty rule and missing outputs are refused up front */
  checl_image* delta = NULL;
  CHECK(checl_checkpoint_incremental_ex(ctx, 0, NULL, 1, img, 2, &delta) == CHECL_ERR_INVALID_VALUE && !delta);
  CHECK(checl_checkpoint_incremental_ex(ctx, 0, NULL, 1, img, CHECL_DIRTY_BYTES, NULL) == CHECL_ERR_INVALID_VALUE);
  CHECK(checl_checkpoint_incremental(ctx, 0, NULL, 1, NULL, &delta) == CHECL_ERR_INVALID_VALUE);
  CHECK(CHECL_DIRTY_CRC == 0 && CHECL_DIRTY_BYTES == 1);
  CHECK(checl_image_free(img) == CHECL_SUCCESS);
  CHECK(checl_image_free(NULL) == CHECL_SUCCESS);
  checl_timing t;
  CHECK(checl_last_timing(ctx, &t) == CHECL_SUCCESS);
  checl_stats st;
  CHECK(checl_stats_get(ctx, CHECL_STATS_RESTORE, &st) == CHECL_SUCCESS && st.n_calls == 0 && st.kernel_ms == 0.0);
  CHECK(checl_stats_get(ctx, CHECL_STATS_KINDS, &st) == CHECL_ERR_INVALID_VALUE);
  CHECK(checl_stats_reset(ctx) == CHECL_SUCCESS);
  CHECK(checl_trim(ctx) == CHECL_SUCCESS); /* nothing kept: no device work */
  CHECK(checl_destroy(ctx) == CHECL_SUCCESS);
  printf("abi_registry ok\n");
  return 0;
}
