// Tensor table / weight-blob layout of the FLUX.1-dev-shaped MMDiT (public architecture; see
// include/tsv.h "Tensor ids").
#include "model.h"

#include <algorithm>

namespace tsv {

namespace {
struct Spec {
  int id;
  std::string name;
  int64_t rows, cols;
  char kind;  // 'w' weight, 'b' bias, 'g' gain
  int64_t fan_in;
};
}  // namespace

bool build_model(const tsv_model_desc& d, Model* m, std::string* err) {
  if (d.hidden <= 0 || d.heads <= 0 || d.head_dim <= 0 || d.hidden != d.heads * d.head_dim) {
    *err = "model: hidden must equal heads * head_dim";
    return false;
  }
  if (d.head_dim != 64 && d.head_dim != 128) { *err = "model: head_dim must be 64 or 128"; return false; }
  if (d.family != TSV_FAMILY_FLUX && d.family != TSV_FAMILY_SD3) { *err = "model: unknown family"; return false; }
  const bool sd3 = d.family == TSV_FAMILY_SD3;
  if (sd3 && (d.n_single != 0 || d.n_double < 1 || d.pe_max <= 0 || d.pe_base <= 0 || d.hidden % 4)) {
    *err = "model: SD3 needs joint blocks only (n_single = 0, n_double >= 1) and pe_max, pe_base > 0";
    return false;
  }
  if (!sd3 && (d.axes_dim[0] + d.axes_dim[1] + d.axes_dim[2] != d.head_dim ||
               (d.axes_dim[0] | d.axes_dim[1] | d.axes_dim[2]) & 1)) {
    *err = "model: axes_dim must be even and sum to head_dim";
    return false;
  }
  if (d.hidden % 128 || d.mlp_hidden % 128 || d.in_ch % 64 || d.ctx_dim % 64 || d.vec_dim % 64 || d.n_double < 0 ||
      d.n_single < 0 || d.text_tokens < 0 || d.n_double + d.n_single == 0 || d.n_double > 60 || d.n_single > 120) {
    *err = "model: unsupported dimensions (hidden, mlp_hidden % 128; in_ch, ctx_dim, vec_dim % 64)";
    return false;
  }
  m->d = d;
  m->h = d.hidden; m->H = d.heads; m->D = d.head_dim; m->F = d.mlp_hidden; m->in = d.in_ch;
  m->ctx = d.ctx_dim; m->vec = d.vec_dim; m->Lt = d.text_tokens;
  const int64_t h = m->h, F = m->F, D = m->D, in = m->in;
  m->sd3 = sd3;
  m->B = sd3 ? 2 : 1;
  m->n_mod = (12 * (int64_t)d.n_double + 3 * (int64_t)d.n_single + 2 - (sd3 ? 4 : 0)) * h;
  m->mod_final_off = m->n_mod - 2 * h;

  std::vector<Spec> specs = {
      {0, "img_in.w", h, in, 'w', in}, {1, "img_in.b", h, 1, 'b', 0},
      {2, "txt_in.w", h, m->ctx, 'w', m->ctx}, {3, "txt_in.b", h, 1, 'b', 0},
      {4, "time_in.in.w", h, 256, 'w', 256}, {5, "time_in.in.b", h, 1, 'b', 0},
      {6, "time_in.out.w", h, h, 'w', h}, {7, "time_in.out.b", h, 1, 'b', 0},
      {8, "guidance_in.in.w", h, 256, 'w', 256}, {9, "guidance_in.in.b", h, 1, 'b', 0},
      {10, "guidance_in.out.w", h, h, 'w', h}, {11, "guidance_in.out.b", h, 1, 'b', 0},
      {12, "vector_in.in.w", h, m->vec, 'w', m->vec}, {13, "vector_in.in.b", h, 1, 'b', 0},
      {14, "vector_in.out.w", h, h, 'w', h}, {15, "vector_in.out.b", h, 1, 'b', 0},
      {16, "final.mod.w", 2 * h, h, 'w', h}, {17, "final.mod.b", 2 * h, 1, 'b', 0},
      {18, "final.lin.w", in, h, 'w', h}, {19, "final.lin.b", in, 1, 'b', 0},
  };
  if (sd3) {  // no guidance embedder
    specs.erase(std::remove_if(specs.begin(), specs.end(), [](const Spec& x) { return x.id >= 8 && x.id <= 11; }),
                specs.end());
  }
  for (int j = 0; j < d.n_double; ++j)
    for (int s = 0; s < 2; ++s) {
      const int b = double_base(j, s);
      const std::string p = (sd3 ? "joint" : "double") + std::to_string(j) + (s ? ".txt." : ".img.");
      if (sd3 && s == 1 && j == d.n_double - 1) {  // context_pre_only: AdaLayerNormContinuous + QKV only
        specs.push_back({b + 0, p + "mod.w", 2 * h, h, 'w', h});
        specs.push_back({b + 1, p + "mod.b", 2 * h, 1, 'b', 0});
        specs.push_back({b + 2, p + "qkv.w", 3 * h, h, 'w', h});
        specs.push_back({b + 3, p + "qkv.b", 3 * h, 1, 'b', 0});
        continue;
      }
      specs.push_back({b + 0, p + "mod.w", 6 * h, h, 'w', h});
      specs.push_back({b + 1, p + "mod.b", 6 * h, 1, 'b', 0});
      specs.push_back({b + 2, p + "qkv.w", 3 * h, h, 'w', h});
      specs.push_back({b + 3, p + "qkv.b", 3 * h, 1, 'b', 0});
      if (!sd3) {
        specs.push_back({b + 4, p + "q_norm.g", D, 1, 'g', 0});
        specs.push_back({b + 5, p + "k_norm.g", D, 1, 'g', 0});
      }
      specs.push_back({b + 6, p + "proj.w", h, h, 'w', h});
      specs.push_back({b + 7, p + "proj.b", h, 1, 'b', 0});
      specs.push_back({b + 8, p + "fc1.w", F, h, 'w', h});
      specs.push_back({b + 9, p + "fc1.b", F, 1, 'b', 0});
      specs.push_back({b + 10, p + "fc2.w", h, F, 'w', F});
      specs.push_back({b + 11, p + "fc2.b", h, 1, 'b', 0});
    }
  for (int j = 0; j < d.n_single; ++j) {
    const int b = single_base(j);
    const std::string p = "single" + std::to_string(j) + ".";
    specs.push_back({b + 0, p + "mod.w", 3 * h, h, 'w', h});
    specs.push_back({b + 1, p + "mod.b", 3 * h, 1, 'b', 0});
    specs.push_back({b + 2, p + "lin1.w", 3 * h + F, h, 'w', h});
    specs.push_back({b + 3, p + "lin1.b", 3 * h + F, 1, 'b', 0});
    specs.push_back({b + 4, p + "q_norm.g", D, 1, 'g', 0});
    specs.push_back({b + 5, p + "k_norm.g", D, 1, 'g', 0});
    specs.push_back({b + 6, p + "lin2.w", h, h + F, 'w', h + F});
    specs.push_back({b + 7, p + "lin2.b", h, 1, 'b', 0});
  }
  int max_id = 0;
  for (auto& s : specs) max_id = s.id > max_id ? s.id : max_id;
  m->by_id.assign(max_id + 1, -1);
  m->tensors.clear();
  for (auto& s : specs) {
    TensorInfo t;
    t.id = s.id; t.name = s.name; t.rows = s.rows; t.cols = s.cols;
    if (s.kind == 'w') { t.kind = SK_BF16; t.c = synth_scale(1.0 / std::sqrt((double)s.fan_in)); }
    else if (s.kind == 'b') { t.kind = SK_BF16; t.c = synth_scale(0.02); }
    else { t.kind = SK_GAIN; t.c = synth_scale(0.1); }
    t.offset = 0;
    m->by_id[s.id] = (int)m->tensors.size();
    m->tensors.push_back(t);
  }
  // layout: modulation weights (table order), modulation biases (table order), the rest
  auto align = [](size_t x) { return (x + 127) & ~size_t(127); };
  std::vector<int> mod_w_ids, mod_b_ids;
  for (int j = 0; j < d.n_double; ++j)
    for (int s = 0; s < 2; ++s) { mod_w_ids.push_back(double_base(j, s)); mod_b_ids.push_back(double_base(j, s) + 1); }
  for (int j = 0; j < d.n_single; ++j) { mod_w_ids.push_back(single_base(j)); mod_b_ids.push_back(single_base(j) + 1); }
  mod_w_ids.push_back(16);
  mod_b_ids.push_back(17);
  size_t off = 0;
  m->modw_off = off;
  for (int id : mod_w_ids) { auto& t = m->tensors[m->by_id[id]]; t.offset = off; off += t.numel(); }
  off = align(off);
  m->modb_off = off;
  for (int id : mod_b_ids) { auto& t = m->tensors[m->by_id[id]]; t.offset = off; off += t.numel(); }
  off = align(off);
  for (auto& t : m->tensors) {
    bool is_mod = false;
    for (int id : mod_w_ids) is_mod |= (id == t.id);
    for (int id : mod_b_ids) is_mod |= (id == t.id);
    if (is_mod) continue;
    t.offset = off;
    off = align(off + t.numel());
  }
  m->total = off;
  return true;
}

}  // namespace tsv
