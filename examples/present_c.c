/*
 * present_c.c -- the C ABI (include/snn.h) used from plain C, no Python and no PyTorch: create a network
 * with a Table I preset, present a batch of images with learning on ("Each image is presented to
 * the network for t_learn ms"), read back the conductance codes, the per-image spike counts, the last output
 * raster and the counters.
 *
 *   usage: present_c N_IN N_EXC BITS PRESET T N_IMAGES images.u8 seeds.u64 out_prefix
 *   writes out_prefix.codes (n_in x n_exc codes, 1 or 2 bytes each; 4-byte binary32 G at 32 bits),
 *          out_prefix.counts (n_images int32), out_prefix.raster (T x ceil(n_exc/32) u32), out_prefix.stats
 *
 * Build: gcc -std=c99 -Wall -Iinclude examples/present_c.c -Lpaper_conf_date_shelm19_b200 -lsnn_b200 \
 *            -Wl,-rpath,$PWD/paper_conf_date_shelm19_b200 -o present_c
 */
#include <stdio.h>
#include <stdlib.h>
#include <stdint.h>
#include "snn.h"

static void* read_file(const char* path, size_t n) {
  FILE* f = fopen(path, "rb");
  if (!f) { perror(path); exit(2); }
  void* buf = malloc(n ? n : 1);
  if (fread(buf, 1, n, f) != n) { fprintf(stderr, "%s: short read\n", path); exit(2); }
  fclose(f);
  return buf;
}

static void write_file(const char* prefix, const char* ext, const void* buf, size_t n) {
  char path[4096];
  snprintf(path, sizeof(path), "%s.%s", prefix, ext);
  FILE* f = fopen(path, "wb");
  if (!f || fwrite(buf, 1, n, f) != n) { perror(path); exit(2); }
  fclose(f);
}

#define CHECK(call)                                                                 \
  do {                                                                              \
    int rc_ = (call);                                                               \
    if (rc_ != SNN_OK) {                                                            \
      fprintf(stderr, "%s failed: %d (%s)\n", #call, rc_, snn_last_error());        \
      return 1;                                                                     \
    }                                                                               \
  } while (0)

int main(int argc, char** argv) {
  if (argc != 10) {
    fprintf(stderr, "usage: %s N_IN N_EXC BITS PRESET T N_IMAGES images.u8 seeds.u64 out_prefix\n", argv[0]);
    return 2;
  }
  const int n_in = atoi(argv[1]), n_exc = atoi(argv[2]), bits = atoi(argv[3]), preset = atoi(argv[4]);
  const int T = atoi(argv[5]), n_images = atoi(argv[6]);
  uint8_t* images = (uint8_t*)read_file(argv[7], (size_t)n_images * n_in);
  uint64_t* seeds = (uint64_t*)read_file(argv[8], sizeof(uint64_t) * (size_t)n_images);

  snn_params p;
  CHECK(snn_params_preset(&p, preset));
  snn_handle* h = NULL;
  CHECK(snn_create(n_in, n_exc, bits, &p, &h));
  int32_t* counts = (int32_t*)calloc((size_t)n_images, sizeof(int32_t));
  CHECK(snn_present_batch(h, images, n_images, T, seeds, counts, 0));   /* host buffers: copies inside */

  const size_t cb = bits == 32 ? 4 : (bits > 8 ? 2 : 1);
  const size_t ncode = (size_t)n_in * n_exc * cb;
  uint8_t* codes = (uint8_t*)malloc(ncode);
  CHECK(snn_get_weights(h, codes, ncode));
  const size_t nr = (size_t)T * ((n_exc + 31) / 32);
  uint32_t* raster = (uint32_t*)calloc(nr ? nr : 1, sizeof(uint32_t));
  CHECK(snn_get_spikes(h, raster, nr));
  uint64_t stats[SNN_NSTATS];
  CHECK(snn_get_stats(h, stats));

  write_file(argv[9], "codes", codes, ncode);
  write_file(argv[9], "counts", counts, sizeof(int32_t) * (size_t)n_images);
  write_file(argv[9], "raster", raster, sizeof(uint32_t) * nr);
  write_file(argv[9], "stats", stats, sizeof(stats));
  long total = 0;
  for (int k = 0; k < n_images; ++k) total += counts[k];
  printf("present_c: %d images, %ld post spikes, %llu input spikes, %llu LTD / %llu LTP events\n", n_images, total,
         (unsigned long long)stats[0], (unsigned long long)stats[3], (unsigned long long)stats[5]);
  CHECK(snn_destroy(h));
  free(images); free(seeds); free(counts); free(codes); free(raster);
  return 0;
}
