// pack.cpp — boundary ingest: residue encoding, the default
// substitution matrix, and the length-sorted interleaved packing of the database.
//
// a1 "Encode + index": the paper converts the flat files once at the master into an
//    indexed format (P16 §IV "converts the format to a more suitable one"; P20 §IV.B
//    "the total number of sequences, the size of the biggest sequence and the offset
//    that marks the beginning of each sequence").  sw_seqset is that format; here the
//    residues become 5-bit codes in NCBI order.
// a2 "Length sort + interleaved packing" (north_star): stable sort by length
//    (descending), groups of 32 sequences (one per lane of a K1 block), each group
//    padded to its longest member rounded up to 8 columns (one K1 tile; the last
//    16-column word may be half used), interleaved so word w of
//    lane l is packed[word_off + w*32 + l] (a warp load = 512 contiguous bytes).
#include <algorithm>
#include <cstring>
#include <numeric>
#include <sstream>
#include <mutex>
#include "sw_internal.h"
#include "../../include/sw.h"

namespace sw {

static const char kAlphabet[] = "ARNDCQEGHILKMFPSTWYVBZX*";

int encode_residue(int c) {
  static int8_t table[256];
  static std::once_flag once;
  std::call_once(once, [] {
    for (int i = 0; i < 256; i++) table[i] = -1;
    for (int k = 0; k < 24; k++) {
      table[(unsigned char)kAlphabet[k]] = (int8_t)k;
      if (kAlphabet[k] >= 'A' && kAlphabet[k] <= 'Z')
        table[(unsigned char)(kAlphabet[k] - 'A' + 'a')] = (int8_t)k;
    }
  });
  return table[c & 0xff];
}

// BLOSUM62 in the NCBI text layout (reading R1), transcribed for libsw independently of
// the oracle's copy and parsed once.  tests/test_native.py checks both copies against
// the checksums of SURVEY §8(c) item 1 and against each other.
static const char kBlosum62Text[] =
    "   A  R  N  D  C  Q  E  G  H  I  L  K  M  F  P  S  T  W  Y  V  B  Z  X  *\n"
    "A  4 -1 -2 -2  0 -1 -1  0 -2 -1 -1 -1 -1 -2 -1  1  0 -3 -2  0 -2 -1  0 -4\n"
    "R -1  5  0 -2 -3  1  0 -2  0 -3 -2  2 -1 -3 -2 -1 -1 -3 -2 -3 -1  0 -1 -4\n"
    "N -2  0  6  1 -3  0  0  0  1 -3 -3  0 -2 -3 -2  1  0 -4 -2 -3  3  0 -1 -4\n"
    "D -2 -2  1  6 -3  0  2 -1 -1 -3 -4 -1 -3 -3 -1  0 -1 -4 -3 -3  4  1 -1 -4\n"
    "C  0 -3 -3 -3  9 -3 -4 -3 -3 -1 -1 -3 -1 -2 -3 -1 -1 -2 -2 -1 -3 -3 -2 -4\n"
    "Q -1  1  0  0 -3  5  2 -2  0 -3 -2  1  0 -3 -1  0 -1 -2 -1 -2  0  3 -1 -4\n"
    "E -1  0  0  2 -4  2  5 -2  0 -3 -3  1 -2 -3 -1  0 -1 -3 -2 -2  1  4 -1 -4\n"
    "G  0 -2  0 -1 -3 -2 -2  6 -2 -4 -4 -2 -3 -3 -2  0 -2 -2 -3 -3 -1 -2 -1 -4\n"
    "H -2  0  1 -1 -3  0  0 -2  8 -3 -3 -1 -2 -1 -2 -1 -2 -2  2 -3  0  0 -1 -4\n"
    "I -1 -3 -3 -3 -1 -3 -3 -4 -3  4  2 -3  1  0 -3 -2 -1 -3 -1  3 -3 -3 -1 -4\n"
    "L -1 -2 -3 -4 -1 -2 -3 -4 -3  2  4 -2  2  0 -3 -2 -1 -2 -1  1 -4 -3 -1 -4\n"
    "K -1  2  0 -1 -3  1  1 -2 -1 -3 -2  5 -1 -3 -1  0 -1 -3 -2 -2  0  1 -1 -4\n"
    "M -1 -1 -2 -3 -1  0 -2 -3 -2  1  2 -1  5  0 -2 -1 -1 -1 -1  1 -3 -1 -1 -4\n"
    "F -2 -3 -3 -3 -2 -3 -3 -3 -1  0  0 -3  0  6 -4 -2 -2  1  3 -1 -3 -3 -1 -4\n"
    "P -1 -2 -2 -1 -3 -1 -1 -2 -2 -3 -3 -1 -2 -4  7 -1 -1 -4 -3 -2 -2 -1 -2 -4\n"
    "S  1 -1  1  0 -1  0  0  0 -1 -2 -2  0 -1 -2 -1  4  1 -3 -2 -2  0  0  0 -4\n"
    "T  0 -1  0 -1 -1 -1 -1 -2 -2 -1 -1 -1 -1 -2 -1  1  5 -2 -2  0 -1 -1  0 -4\n"
    "W -3 -3 -4 -4 -2 -2 -3 -2 -2 -3 -2 -3 -1  1 -4 -3 -2 11  2 -3 -4 -3 -2 -4\n"
    "Y -2 -2 -2 -3 -2 -1 -2 -3  2 -1 -1 -2 -1  3 -3 -2 -2  2  7 -1 -3 -2 -1 -4\n"
    "V  0 -3 -3 -3 -1 -2 -2 -3 -3  3  1 -2  1 -1 -2 -2  0 -3 -1  4 -3 -2 -1 -4\n"
    "B -2 -1  3  4 -3  0  1 -1  0 -3 -4  0 -3 -3 -2  0 -1 -4 -3 -3  4  1 -1 -4\n"
    "Z -1  0  0  1 -3  3  4 -2  0 -3 -3  1 -1 -3 -1  0 -1 -3 -2 -2  1  4 -1 -4\n"
    "X  0 -1 -1 -1 -2 -1 -1 -1 -1 -1 -1 -1 -1 -1 -2  0  0 -2 -1 -1 -1 -1 -1 -4\n"
    "* -4 -4 -4 -4 -4 -4 -4 -4 -4 -4 -4 -4 -4 -4 -4 -4 -4 -4 -4 -4 -4 -4 -4  1\n";

const int8_t *blosum62() {
  static int8_t m[24 * 24];
  static std::once_flag once;
  std::call_once(once, [] {
    std::istringstream in(kBlosum62Text);
    std::string line;
    std::getline(in, line);  // header: column letters in alphabet order
    std::vector<int> col;
    for (char ch : line)
      if (ch != ' ') col.push_back(encode_residue(ch));
    while (std::getline(in, line)) {
      std::istringstream ls(line);
      std::string row;
      ls >> row;
      int r = encode_residue(row[0]);
      for (int k = 0; k < 24; k++) {
        int v;
        ls >> v;
        m[r * 24 + col[k]] = (int8_t)v;
      }
    }
  });
  return m;
}

// database residue code -> slot (sw_internal.h: SW_CODE_OF_SLOT_INIT, inverted)
static const struct SlotTable {
  uint8_t v[kNCodes];
  SlotTable() {
    const uint8_t code_of_slot[kNCodes] = SW_CODE_OF_SLOT_INIT;
    for (int sl = 0; sl < kNCodes; sl++) v[code_of_slot[sl]] = (uint8_t)sl;
  }
} slot_table;
static const uint8_t *const slot_of_code = slot_table.v;

int pack_database(const int64_t *offsets, const char *residues, int32_t n, PackedDB &out,
                  std::string &err) {
  out = PackedDB();
  out.n = n;
  if (n < 0) { err = "db: n < 0"; return SW_EINVAL; }
  if (n == 0) return SW_OK;
  if (!offsets) { err = "db: offsets is NULL"; return SW_EINVAL; }
  if (offsets[0] != 0) { err = "db: offsets[0] != 0"; return SW_EINVAL; }
  std::vector<int32_t> len(n);
  for (int32_t k = 0; k < n; k++) {
    int64_t l = offsets[k + 1] - offsets[k];
    if (l < 0) { err = "db: offsets not monotone at sequence " + std::to_string(k); return SW_EINVAL; }
    if (l > (1 << 30)) { err = "db: sequence too long at " + std::to_string(k); return SW_EINVAL; }
    len[k] = (int32_t)l;
  }
  out.residues = offsets[n];
  if (out.residues > 0 && !residues) { err = "db: residues is NULL"; return SW_EINVAL; }
  // validate every residue (strict alphabet)
  for (int32_t k = 0; k < n; k++)
    for (int64_t p = offsets[k]; p < offsets[k + 1]; p++)
      if (encode_residue((unsigned char)residues[p]) < 0) {
        err = "db: invalid residue '" + std::string(1, residues[p]) + "' in sequence " +
              std::to_string(k) + " at position " + std::to_string(p - offsets[k]);
        return SW_ERESIDUE;
      }
  // stable sort by length, descending (longest first: LPT order)
  out.perm.resize(n);
  std::iota(out.perm.begin(), out.perm.end(), 0);
  std::stable_sort(out.perm.begin(), out.perm.end(),
                   [&](int32_t a, int32_t b) { return len[a] > len[b]; });
  out.sorted_len.resize(n);
  for (int32_t s = 0; s < n; s++) out.sorted_len[s] = len[out.perm[s]];
  out.max_len = out.sorted_len[0];
  // groups and interleaved words
  const int32_t ng = (n + kGroup - 1) / kGroup;
  out.groups.resize(ng);
  int64_t words = 0;
  for (int32_t g = 0; g < ng; g++) {
    GroupInfo &G = out.groups[g];
    G.first = g * kGroup;
    G.count = std::min(kGroup, n - G.first);
    int32_t l = out.sorted_len[G.first];
    int32_t cols = (l + kColAlign - 1) / kColAlign * kColAlign;
    G.ncols = std::max(cols, kMinCols);
    G.word_off = words;
    G.pad_ = 0;
    words += (int64_t)((G.ncols + kWordCols - 1) / kWordCols) * kGroup;
  }
  out.packed.assign(words, make_uint4(0, 0, 0, 0));
  uint8_t *bytes = reinterpret_cast<uint8_t *>(out.packed.data());
  for (int32_t g = 0; g < ng; g++) {
    const GroupInfo &G = out.groups[g];
    const int32_t nw = (G.ncols + kWordCols - 1) / kWordCols;
    for (int32_t lane = 0; lane < kGroup; lane++) {
      const int32_t s = G.first + lane;
      const bool real = lane < G.count;
      const char *src = real ? residues + offsets[out.perm[s]] : nullptr;
      const int32_t l = real ? out.sorted_len[s] : 0;
      for (int32_t w = 0; w < nw; w++) {
        uint8_t *dst = bytes + ((G.word_off + (int64_t)w * kGroup + lane) * 16);
        for (int b = 0; b < kWordCols; b++) {
          int32_t j = w * kWordCols + b;
          dst[b] = (j < l) ? slot_of_code[encode_residue((unsigned char)src[j])] : (uint8_t)kPadCode;
        }
      }
    }
  }
  return SW_OK;
}

}  // namespace sw
