// Host harness for tests/test_pack_swar.py: reads raw records (uint32[n][9]) from the file
// argv[1], writes the packed rows (uint32[n][4]) that the product's pack_record
// (paper_conf_asplos_finglertyshar23_b200/csrc/digitize.cuh, __host__ __device__) produces
// to argv[2]. Host-side only: no GPU needed; the test unpacks the nibbles and compares them
// with the oracle's digits.
#include <cstdio>
#include <vector>

#include "../paper_conf_asplos_finglertyshar23_b200/csrc/digitize.cuh"

int main(int argc, char **argv) {
  if (argc != 3) return 2;
  FILE *f = std::fopen(argv[1], "rb");
  if (!f) return 3;
  std::vector<uint32_t> raw;
  uint32_t buf[9];
  while (std::fread(buf, 4, 9, f) == 9) raw.insert(raw.end(), buf, buf + 9);
  std::fclose(f);
  const size_t n = raw.size() / 9;
  std::vector<uint32_t> out(n * 4);
  for (size_t i = 0; i < n; ++i) {
    uint32_t rec[9];
    for (int k = 0; k < 9; ++k) rec[k] = raw[i * 9 + k];
    const uint4 p = lake::pack_record(rec);
    out[i * 4 + 0] = p.x; out[i * 4 + 1] = p.y; out[i * 4 + 2] = p.z; out[i * 4 + 3] = p.w;
  }
  FILE *g = std::fopen(argv[2], "wb");
  if (!g) return 4;
  std::fwrite(out.data(), 4, out.size(), g);
  std::fclose(g);
  return 0;
}
