// Model registration and the pinned host weight arena.
//
// "To optimize data transfers from the host to GPU, we allocate the pinned memory
// for the layers.  For layers executed by direct-host-access, we add a new memory
// allocator in PyTorch that allocates memory through cudaHostAlloc."  Here every layer
// lives in ONE cudaHostAlloc(Portable | Mapped) arena: mapped so any unit can be read in
// place by a DHA kernel, portable so every GPU of the context can DMA from it, packed in
// forward order with 256-byte aligned units so a run of adjacent loaded units is one
// contiguous DMA.  Planning units follow SURVEY G1 (one weight-bearing leaf module).
#include "engine.h"
#include "model.h"

#include <cstring>

namespace dp {

void validate_config(const dp_model_config& c) {
  DP_CHECK(c.family == DP_FAMILY_BERT || c.family == DP_FAMILY_ROBERTA || c.family == DP_FAMILY_GPT2,
           DP_ERR_INVALID, "unknown model family");
  DP_CHECK(c.dtype == DP_FP16 || c.dtype == DP_BF16 || c.dtype == DP_FP32, DP_ERR_UNSUPPORTED,
           "dtype must be fp16, bf16 or fp32");
  DP_CHECK(c.hidden > 0 && c.hidden % 64 == 0, DP_ERR_INVALID, "hidden must be a positive multiple of 64");
  DP_CHECK(c.heads > 0 && c.hidden % c.heads == 0, DP_ERR_INVALID, "hidden % heads != 0");
  DP_CHECK(c.ffn > 0 && c.ffn % 64 == 0, DP_ERR_INVALID, "ffn must be a positive multiple of 64");
  DP_CHECK(c.vocab > 0 && c.max_pos > 0 && c.layers >= 0, DP_ERR_INVALID, "bad vocab/max_pos/layers");
  DP_CHECK(c.family == DP_FAMILY_GPT2 || c.type_vocab > 0, DP_ERR_INVALID, "type_vocab must be > 0");
  DP_CHECK(c.ln_eps > 0, DP_ERR_INVALID, "ln_eps must be > 0");
}

std::vector<ParamDesc> config_params(const dp_model_config& c) {
  validate_config(c);
  std::vector<ParamDesc> ps;
  const int64_t H = c.hidden, F = c.ffn;
  auto add = [&](const std::string& name, int64_t a, int64_t b = -1, bool tr = false) {
    ParamDesc p;
    p.hf = name;
    p.ndim = b < 0 ? 1 : 2;
    p.shape[0] = a;
    p.shape[1] = b < 0 ? 0 : b;
    p.bytes = a * (b < 0 ? 1 : b) * dtype_bytes(c.dtype);
    p.transpose = tr;
    ps.push_back(p);
  };
  if (c.family != DP_FAMILY_GPT2) {
    add("embeddings.word_embeddings.weight", c.vocab, H);
    add("embeddings.position_embeddings.weight", c.max_pos, H);
    add("embeddings.token_type_embeddings.weight", c.type_vocab, H);
    add("embeddings.LayerNorm.weight", H);
    add("embeddings.LayerNorm.bias", H);
    for (int l = 0; l < c.layers; ++l) {
      const std::string p = "encoder.layer." + std::to_string(l) + ".";
      for (const char* nm : {"query", "key", "value"}) {
        add(p + "attention.self." + nm + ".weight", H, H);
        add(p + "attention.self." + nm + ".bias", H);
      }
      add(p + "attention.output.dense.weight", H, H);
      add(p + "attention.output.dense.bias", H);
      add(p + "attention.output.LayerNorm.weight", H);
      add(p + "attention.output.LayerNorm.bias", H);
      add(p + "intermediate.dense.weight", F, H);
      add(p + "intermediate.dense.bias", F);
      add(p + "output.dense.weight", H, F);
      add(p + "output.dense.bias", H);
      add(p + "output.LayerNorm.weight", H);
      add(p + "output.LayerNorm.bias", H);
    }
    add("pooler.dense.weight", H, H);
    add("pooler.dense.bias", H);
  } else {
    add("wte.weight", c.vocab, H);
    add("wpe.weight", c.max_pos, H);
    for (int l = 0; l < c.layers; ++l) {
      const std::string p = "h." + std::to_string(l) + ".";
      add(p + "ln_1.weight", H);
      add(p + "ln_1.bias", H);
      add(p + "attn.c_attn.weight", H, 3 * H, true);
      add(p + "attn.c_attn.bias", 3 * H);
      add(p + "attn.c_proj.weight", H, H, true);
      add(p + "attn.c_proj.bias", H);
      add(p + "ln_2.weight", H);
      add(p + "ln_2.bias", H);
      add(p + "mlp.c_fc.weight", H, F, true);
      add(p + "mlp.c_fc.bias", F);
      add(p + "mlp.c_proj.weight", F, H, true);
      add(p + "mlp.c_proj.bias", H);
    }
    add("ln_f.weight", H);
    add("ln_f.bias", H);
  }
  return ps;
}

void build_units(dp_model* m) {
  const auto& c = m->cfg;
  auto& U = m->units;
  int pi = 0;
  auto unit = [&](const std::string& name, int kind, int role, int layer, int np, int64_t N = 0, int64_t K = 0) {
    UnitDesc u;
    u.name = name;
    u.kind = kind;
    u.role = role;
    u.layer = layer;
    u.first_param = pi;
    u.nparams = np;
    u.N = N;
    u.K = K;
    for (int j = 0; j < np; ++j) {
      m->params[pi + j].unit = (int)U.size();
      u.bytes += m->params[pi + j].bytes;
    }
    pi += np;
    U.push_back(u);
  };
  const int64_t H = c.hidden, F = c.ffn;
  if (c.family != DP_FAMILY_GPT2) {
    unit("word", DP_UNIT_EMB, R_WORD, -1, 1);
    unit("pos", DP_UNIT_EMB, R_POS, -1, 1);
    unit("type", DP_UNIT_EMB, R_TYPE, -1, 1);
    unit("emb_ln", DP_UNIT_LN, R_EMB_LN, -1, 2);
    for (int l = 0; l < c.layers; ++l) {
      const std::string p = "L" + std::to_string(l) + ".";
      unit(p + "q", DP_UNIT_LINEAR, R_Q, l, 2, H, H);
      unit(p + "k", DP_UNIT_LINEAR, R_K, l, 2, H, H);
      unit(p + "v", DP_UNIT_LINEAR, R_V, l, 2, H, H);
      unit(p + "attn_out", DP_UNIT_LINEAR, R_ATTN_OUT, l, 2, H, H);
      unit(p + "ln1", DP_UNIT_LN, R_LN1, l, 2);
      unit(p + "fc1", DP_UNIT_LINEAR, R_FC1, l, 2, F, H);
      unit(p + "fc2", DP_UNIT_LINEAR, R_FC2, l, 2, H, F);
      unit(p + "ln2", DP_UNIT_LN, R_LN2, l, 2);
    }
    unit("pooler", DP_UNIT_LINEAR, R_POOLER, -1, 2, H, H);
  } else {
    unit("wte", DP_UNIT_EMB, R_WTE, -1, 1);
    unit("wpe", DP_UNIT_EMB, R_WPE, -1, 1);
    for (int l = 0; l < c.layers; ++l) {
      const std::string p = "L" + std::to_string(l) + ".";
      unit(p + "ln_1", DP_UNIT_LN, R_LN_1, l, 2);
      unit(p + "c_attn", DP_UNIT_LINEAR, R_C_ATTN, l, 2, 3 * H, H);
      unit(p + "c_proj", DP_UNIT_LINEAR, R_C_PROJ, l, 2, H, H);
      unit(p + "ln_2", DP_UNIT_LN, R_LN_2, l, 2);
      unit(p + "c_fc", DP_UNIT_LINEAR, R_C_FC, l, 2, F, H);
      unit(p + "mlp_c_proj", DP_UNIT_LINEAR, R_MLP_PROJ, l, 2, H, F);
    }
    unit("ln_f", DP_UNIT_LN, R_LN_F, -1, 2);
  }
  // arena layout: units in forward order, 256-byte aligned; params packed inside a unit
  int64_t off = 0;
  for (auto& u : U) {
    off = (off + 255) & ~int64_t(255);
    u.off = off;
    int64_t po = off;
    for (int j = 0; j < u.nparams; ++j) {
      m->params[u.first_param + j].off = po;
      po += m->params[u.first_param + j].bytes;
    }
    off = po;
  }
  m->arena_bytes = (off + 4095) & ~int64_t(4095);
}

}  // namespace dp

using namespace dp;

extern "C" dp_status dp_config_params(const dp_model_config* cfg, dp_param_info* infos, int32_t cap, int32_t* count) {
  return guard([&] {
    DP_CHECK(cfg && count, DP_ERR_INVALID, "NULL argument");
    dp_model tmp;
    tmp.cfg = *cfg;
    tmp.params = config_params(*cfg);
    build_units(&tmp);
    *count = (int32_t)tmp.params.size();
    for (int i = 0; infos && i < cap && i < (int)tmp.params.size(); ++i) {
      const auto& p = tmp.params[i];
      std::memset(&infos[i], 0, sizeof(dp_param_info));
      std::strncpy(infos[i].hf_name, p.hf.c_str(), sizeof(infos[i].hf_name) - 1);
      infos[i].ndim = p.ndim;
      infos[i].unit = p.unit;
      infos[i].shape[0] = p.shape[0];
      infos[i].shape[1] = p.shape[1];
      infos[i].bytes = p.bytes;
    }
  });
}

extern "C" dp_status dp_model_create(dp_context* ctx, const dp_model_config* cfg, const void* const* host_params,
                                     int32_t nparams, dp_model** out) {
  dp_model* m = nullptr;
  dp_status st = guard([&] {
    DP_CHECK(cfg && out && host_params, DP_ERR_INVALID, "NULL argument");
    m = new dp_model();
    m->cfg = *cfg;
    m->params = config_params(*cfg);
    DP_CHECK(nparams == (int32_t)m->params.size(), DP_ERR_INVALID,
             "expected " + std::to_string(m->params.size()) + " parameters, got " + std::to_string(nparams));
    build_units(m);
    // the arena lives on the NUMA node of the context's first (serving) device: its loads and
    // DHA reads cross no socket interconnect (topo.cpp)
    const int node = (ctx && !ctx->devs.empty()) ? device_numa_node(ctx->devs[0]) : -1;
    m->arena = host_alloc_on_node(m->arena_bytes, node);
    if (!m->arena) fail(DP_ERR_OOM, "cudaHostAlloc of the weight arena failed");
    m->arena_node = node;
    m->arena_owner = std::shared_ptr<void>(m->arena, [](void* p) { cudaFreeHost(p); });
    std::memset(m->arena, 0, m->arena_bytes);
    uint8_t* base = static_cast<uint8_t*>(m->arena);
    for (size_t i = 0; i < m->params.size(); ++i) {
      const auto& p = m->params[i];
      DP_CHECK(host_params[i] != nullptr, DP_ERR_INVALID, "parameter " + p.hf + " is NULL");
      if (!p.transpose) {
        std::memcpy(base + p.off, host_params[i], p.bytes);
      } else {  // [in=a, out=b] -> [out, in]
        const int64_t a = p.shape[0], b = p.shape[1];
        if (dtype_bytes(cfg->dtype) == 4) {
          const uint32_t* src = static_cast<const uint32_t*>(host_params[i]);
          uint32_t* dst = reinterpret_cast<uint32_t*>(base + p.off);
          for (int64_t r = 0; r < a; ++r)
            for (int64_t c = 0; c < b; ++c) dst[c * a + r] = src[r * b + c];
        } else {
          const uint16_t* src = static_cast<const uint16_t*>(host_params[i]);
          uint16_t* dst = reinterpret_cast<uint16_t*>(base + p.off);
          for (int64_t r = 0; r < a; ++r)
            for (int64_t c = 0; c < b; ++c) dst[c * a + r] = src[r * b + c];
        }
      }
    }
    *out = m;
  });
  if (st != DP_OK && m) delete m;  // the arena owner frees the pinned memory
  return st;
}

extern "C" dp_status dp_model_clone(dp_context* ctx, const dp_model* src, dp_model** out) {
  return guard([&] {
    DP_CHECK(src && out, DP_ERR_INVALID, "NULL argument");
    dp_model* m = new dp_model();
    m->cfg = src->cfg;
    m->params = src->params;
    m->units = src->units;
    m->arena = src->arena;
    m->arena_bytes = src->arena_bytes;
    m->arena_owner = src->arena_owner;
    *out = m;
  });
}

extern "C" int32_t dp_model_num_units(const dp_model* m) { return m ? (int32_t)m->units.size() : 0; }

extern "C" dp_status dp_model_unit_info(const dp_model* m, int32_t i, dp_unit_info* out) {
  return guard([&] {
    DP_CHECK(m && out && i >= 0 && i < (int32_t)m->units.size(), DP_ERR_INVALID, "bad unit index");
    const auto& u = m->units[i];
    std::memset(out, 0, sizeof(*out));
    out->kind = u.kind;
    out->nparams = u.nparams;
    out->first_param = u.first_param;
    out->bytes = u.bytes;
    out->arena_offset = u.off;
    std::strncpy(out->name, u.name.c_str(), sizeof(out->name) - 1);
  });
}

extern "C" int64_t dp_model_bytes(const dp_model* m) {
  if (!m) return 0;
  int64_t s = 0;
  for (const auto& u : m->units) s += u.bytes;
  return s;
}

extern "C" dp_status dp_model_arena(const dp_model* m, const void** ptr, int64_t* bytes) {
  return guard([&] {
    DP_CHECK(m && ptr && bytes, DP_ERR_INVALID, "NULL argument");
    *ptr = m->arena;
    *bytes = m->arena_bytes;
  });
}
