// Model description, tensor table and weight-blob layout (host side of libtsv.so).
#pragma once
#include <cmath>
#include <cstdint>
#include <string>
#include <vector>

#include "../../include/tsv.h"

namespace tsv {

enum SynthKind { SK_BF16 = 0, SK_GAIN = 1, SK_F32 = 2 };

struct TensorInfo {
  int id;
  std::string name;
  int64_t rows, cols;  // cols = 1 for vectors
  int kind;            // SynthKind
  float c;             // SYNTH-1 scale constant float32(sqrt(3) * sigma)
  size_t offset;       // elements into the weight blob
  int64_t numel() const { return rows * cols; }
};

inline float synth_scale(double sigma) { return (float)(std::sqrt(3.0) * sigma); }

struct Model {
  tsv_model_desc d{};
  int h = 0, H = 0, D = 0, F = 0, in = 0, ctx = 0, vec = 0, Lt = 0;
  bool sd3 = false;           // TSV_FAMILY_SD3
  int B = 1;                  // transformer evaluations per step: 1, or 2 for SD3's CFG pair
  int64_t n_mod = 0;          // modulation-table width per evaluation: (12 n_double + 3 n_single + 2) h
                              // (SD3: (12 n_double - 4 + 2) h, the last txt stream has 2 chunks)
  int64_t mod_final_off = 0;
  size_t modw_off = 0;        // concatenated modulation weights [n_mod, h]
  size_t modb_off = 0;        // concatenated modulation biases [n_mod]
  size_t total = 0;           // blob elements (bf16)
  std::vector<TensorInfo> tensors;
  std::vector<int> by_id;     // tensor id -> index in tensors (-1 if absent)

  const TensorInfo* find(int id) const {
    return (id >= 0 && id < (int)by_id.size() && by_id[id] >= 0) ? &tensors[by_id[id]] : nullptr;
  }
  // offsets (columns) into one step's modulation row
  int64_t mod_double(int j, int s) const { return (int64_t)j * 12 * h + (int64_t)s * 6 * h; }
  int64_t mod_single(int j) const { return (int64_t)d.n_double * 12 * h + (int64_t)j * 3 * h; }
  int64_t mod_final() const { return mod_final_off; }
};

static inline int double_base(int j, int s) { return 64 + 32 * j + 16 * s; }
static inline int single_base(int j) { return 4096 + 16 * j; }

// Builds the tensor table and the blob layout: modulation weights of every block first, in
// modulation-table order (double j: img, txt; single j; final), then modulation biases, then
// everything else in id order.  Returns false on an invalid description.
bool build_model(const tsv_model_desc& d, Model* m, std::string* err);

}  // namespace tsv
