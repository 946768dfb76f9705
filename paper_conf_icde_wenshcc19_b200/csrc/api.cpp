// api.cpp -- the extern "C" boundary of libgmpsvm.so (include/gmpsvm.h).
// Converts engine exceptions into status codes + a thread-local message; implements the
// model introspection and the serialize / deserialize / merge plumbing used by the
// multi-GPU driver (pairs sharded across ranks, blobs gathered with NCCL).
#include <dlfcn.h>

#include <algorithm>
#include <cstdlib>
#include <cstring>
#include <new>
#include <string>

#include "model.h"

using gmpsvm::Error;
using gmpsvm::Model;

namespace {

// The solver runs every pair's outer loop as its own branch of one CUDA graph; the runtime
// executes at most CUDA_DEVICE_MAX_CONNECTIONS (default 8, max 32) branches concurrently.
// Raise the default to 32 when the library is loaded (an explicit user setting is kept).  The
// variable is read when a CUDA context is created: if the process already has one (e.g. torch
// initialised CUDA before the library was loaded), the setting cannot take effect, so the
// number of connections actually in effect is recorded here and engine.cu packs the pairs into
// that many branches.  libcuda is only probed if it is already loaded (RTLD_NOLOAD).
int g_conn_effective = 8;
__attribute__((constructor)) void gmpsvm_default_connections() {
  const char* prev = getenv("CUDA_DEVICE_MAX_CONNECTIONS");
  const int want = prev ? atoi(prev) : 32;
  int ctx_active = 0;
  if (void* h = dlopen("libcuda.so.1", RTLD_NOW | RTLD_NOLOAD)) {
    using GetState = int (*)(int, unsigned*, int*);
    if (auto fn = reinterpret_cast<GetState>(dlsym(h, "cuDevicePrimaryCtxGetState"))) {
      unsigned flags = 0;
      int active = 0;
      if (fn(0, &flags, &active) == 0) ctx_active = active;
    }
    dlclose(h);
  }
  if (!prev) setenv("CUDA_DEVICE_MAX_CONNECTIONS", "32", 0);
  // a context created before the load saw the user's value (if any) or the runtime default
  const int eff = ctx_active ? (prev ? want : 8) : want;
  g_conn_effective = std::max(1, std::min(32, eff));
}


thread_local std::string g_err;

template <class F>
int guarded(F&& f) {
  try {
    g_err.clear();
    return f();
  } catch (const Error& e) {
    g_err = e.what();
    return e.code;
  } catch (const std::bad_alloc&) {
    g_err = "host allocation failed";
    return GMPSVM_ENOMEM;
  } catch (const std::exception& e) {
    g_err = e.what();
    return GMPSVM_ECUDA;
  } catch (...) {
    g_err = "unknown error";
    return GMPSVM_ECUDA;
  }
}

gmpsvm_options resolve(const gmpsvm_options* opt) {
  gmpsvm_options o;
  gmpsvm_options_init(&o);
  if (opt) {
    if (opt->struct_size != 0 && opt->struct_size != (int32_t)sizeof(gmpsvm_options))
      throw Error(GMPSVM_EINVAL, "gmpsvm_options.struct_size mismatch");
    o = *opt;
  }
  return o;
}

// ---- serialization (flat little-endian; x86-64 / aarch64 hosts are little-endian) ----
const char kMagic[8] = {'G', 'M', 'P', 'S', 'V', 'M', '0', '1'};

struct Writer {
  std::vector<uint8_t> buf;
  template <class T>
  void put(const T& v) {
    const uint8_t* p = reinterpret_cast<const uint8_t*>(&v);
    buf.insert(buf.end(), p, p + sizeof(T));
  }
  template <class T>
  void put_vec(const std::vector<T>& v) {
    const uint8_t* p = reinterpret_cast<const uint8_t*>(v.data());
    buf.insert(buf.end(), p, p + v.size() * sizeof(T));
  }
};

struct Reader {
  const uint8_t* p;
  size_t left;
  template <class T>
  T get() {
    if (left < sizeof(T)) throw Error(GMPSVM_EFORMAT, "truncated model blob");
    T v;
    std::memcpy(&v, p, sizeof(T));
    p += sizeof(T);
    left -= sizeof(T);
    return v;
  }
  template <class T>
  void get_vec(std::vector<T>& v, size_t count) {
    if (count > left / sizeof(T)) throw Error(GMPSVM_EFORMAT, "truncated model blob");
    v.resize(count);
    std::memcpy(v.data(), p, count * sizeof(T));
    p += count * sizeof(T);
    left -= count * sizeof(T);
  }
};

std::vector<uint8_t> serialize(const Model& m) {
  {
    std::lock_guard<std::mutex> lk(m.mu);
    gmpsvm::ensure_host_sv(m);
    gmpsvm::ensure_host_alpha(m);
  }
  Writer w;
  w.buf.insert(w.buf.end(), kMagic, kMagic + 8);
  w.put<int32_t>(GMPSVM_ABI_VERSION);
  w.put<int32_t>(m.k);
  w.put<int32_t>(m.d);
  w.put<int32_t>(m.kernel);
  w.put<double>(m.C);
  w.put<double>(m.gamma);
  w.put<double>(m.eps);
  w.put<int64_t>(m.n);
  w.put_vec(m.class_count);
  w.put_vec(m.perm);
  w.put_vec(m.trained);
  w.put_vec(m.b);
  w.put_vec(m.A);
  w.put_vec(m.B);
  w.put_vec(m.status);
  w.put_vec(m.alpha);
  w.put<int64_t>((int64_t)m.sv_pos.size());
  w.put_vec(m.sv_pos);
  w.put_vec(m.sv_X);
  w.put(m.stats);
  w.put<double>(m.coef0);
  w.put<int32_t>(m.degree);
  return std::move(w.buf);
}

Model* deserialize(const void* buf, size_t len) {
  if (!buf || len < 8 || std::memcmp(buf, kMagic, 8) != 0) throw Error(GMPSVM_EFORMAT, "not a gmpsvm model blob");
  Reader r{static_cast<const uint8_t*>(buf) + 8, len - 8};
  auto m = std::make_unique<Model>();
  if (r.get<int32_t>() != GMPSVM_ABI_VERSION) throw Error(GMPSVM_EFORMAT, "model blob version mismatch");
  m->k = r.get<int32_t>();
  m->d = r.get<int32_t>();
  m->kernel = r.get<int32_t>();
  if (m->kernel < 0 || m->kernel > 3) throw Error(GMPSVM_EFORMAT, "bad kernel type");
  m->C = r.get<double>();
  m->gamma = r.get<double>();
  m->eps = r.get<double>();
  m->n = r.get<int64_t>();
  if (m->k < 2 || m->k > 64 || m->d < 1 || m->n < 2) throw Error(GMPSVM_EFORMAT, "bad model header");
  const int P = m->P();
  r.get_vec(m->class_count, m->k);
  int64_t tot = 0;
  for (auto c : m->class_count) {
    if (c <= 0) throw Error(GMPSVM_EFORMAT, "bad class counts");
    tot += c;
  }
  if (tot != m->n) throw Error(GMPSVM_EFORMAT, "class counts do not sum to n");
  r.get_vec(m->perm, m->n);
  r.get_vec(m->trained, P);
  r.get_vec(m->b, P);
  r.get_vec(m->A, P);
  r.get_vec(m->B, P);
  r.get_vec(m->status, P);
  r.get_vec(m->alpha, m->pair_offsets()[P]);
  const int64_t nsv = r.get<int64_t>();
  if (nsv < 0 || nsv > m->n) throw Error(GMPSVM_EFORMAT, "bad SV count");
  r.get_vec(m->sv_pos, nsv);
  for (int64_t i = 0; i < nsv; ++i)
    if (m->sv_pos[i] < 0 || m->sv_pos[i] >= m->n || (i && m->sv_pos[i] <= m->sv_pos[i - 1]))
      throw Error(GMPSVM_EFORMAT, "bad SV positions");
  r.get_vec(m->sv_X, (size_t)nsv * m->d);
  m->stats = r.get<gmpsvm_train_stats>();
  m->coef0 = r.get<double>();
  m->degree = r.get<int32_t>();
  m->sv_X_ready = true;
  return m.release();
}

Model* merge(const Model* const* parts, int n) {
  if (n < 1) throw Error(GMPSVM_EINVAL, "no parts");
  const Model& f = *parts[0];
  for (int i = 0; i < n; ++i) {
    const Model& q = *parts[i];
    if (q.k != f.k || q.d != f.d || q.n != f.n || q.C != f.C || q.gamma != f.gamma || q.kernel != f.kernel ||
        q.coef0 != f.coef0 || q.degree != f.degree || q.class_count != f.class_count ||
        q.perm != f.perm)
      throw Error(GMPSVM_EINVAL, "parts were not trained on the same problem");
    std::lock_guard<std::mutex> lk(q.mu);
    gmpsvm::ensure_host_sv(q);
    gmpsvm::ensure_host_alpha(q);
  }
  auto m = std::make_unique<Model>();
  m->k = f.k;
  m->d = f.d;
  m->C = f.C;
  m->gamma = f.gamma;
  m->eps = f.eps;
  m->kernel = f.kernel;
  m->coef0 = f.coef0;
  m->degree = f.degree;
  m->n = f.n;
  m->class_count = f.class_count;
  m->perm = f.perm;
  const int P = f.P();
  m->trained.assign(P, 0);
  m->b.assign(P, 0.0);
  m->A.assign(P, 0.0);
  m->B.assign(P, 0.0);
  m->status.assign(P, 0);
  const auto po = f.pair_offsets();
  m->alpha.assign(po[P], 0.0);
  for (int i = 0; i < n; ++i) {
    const Model& q = *parts[i];
    for (int p = 0; p < P; ++p) {
      if (!q.trained[p]) continue;
      if (m->trained[p]) throw Error(GMPSVM_EINVAL, "pair trained by more than one part");
      m->trained[p] = 1;
      m->b[p] = q.b[p];
      m->A[p] = q.A[p];
      m->B[p] = q.B[p];
      m->status[p] = q.status[p];
      std::copy(q.alpha.begin() + po[p], q.alpha.begin() + po[p + 1], m->alpha.begin() + po[p]);
    }
  }
  // SV union: sorted merge of the parts' SV position lists, rows taken from the first owner
  std::vector<std::pair<int64_t, std::pair<int, int64_t>>> all;
  for (int i = 0; i < n; ++i)
    for (size_t j = 0; j < parts[i]->sv_pos.size(); ++j) all.push_back({parts[i]->sv_pos[j], {i, (int64_t)j}});
  std::sort(all.begin(), all.end());
  for (size_t j = 0; j < all.size(); ++j) {
    if (j && all[j].first == all[j - 1].first) continue;
    m->sv_pos.push_back(all[j].first);
    const Model& q = *parts[all[j].second.first];
    const float* row = q.sv_X.data() + (size_t)all[j].second.second * q.d;
    m->sv_X.insert(m->sv_X.end(), row, row + q.d);
  }
  m->sv_X_ready = true;
  m->stats = f.stats;
  m->stats.n_sv = (int64_t)m->sv_pos.size();
  m->stats.n_pairs_trained = m->n_trained();
  return m.release();
}

}  // namespace

namespace gmpsvm {
int connections_in_effect() { return g_conn_effective; }
}  // namespace gmpsvm

extern "C" {

void gmpsvm_options_init(gmpsvm_options* opt) {
  if (!opt) return;
  std::memset(opt, 0, sizeof(*opt));
  opt->struct_size = (int32_t)sizeof(gmpsvm_options);
}

int gmpsvm_train_ex(const float* X, const int32_t* y, int64_t n, int32_t d, int32_t k, double C, double gamma,
                    double eps, const gmpsvm_options* opt, gmpsvm_model** out) {
  return guarded([&]() {
    if (!out) throw Error(GMPSVM_EINVAL, "out is NULL");
    *out = nullptr;
    const gmpsvm_options o = resolve(opt);
    Model* m = nullptr;
    const int rc = gmpsvm::engine_train(X, y, n, d, k, C, gamma, eps, o, &m);
    auto* h = new gmpsvm_model();
    h->m.reset(m);
    *out = h;
    return rc;
  });
}

int gmpsvm_train(const float* X, const int32_t* y, int64_t n, int32_t d, int32_t k, double C, double gamma, double eps,
                 gmpsvm_model** out) {
  return gmpsvm_train_ex(X, y, n, d, k, C, gamma, eps, nullptr, out);
}

int gmpsvm_predict_proba_ex(const gmpsvm_model* model, const float* Xtest, int64_t m, double* out,
                            const gmpsvm_options* opt) {
  return guarded([&]() {
    if (!model) throw Error(GMPSVM_EINVAL, "model is NULL");
    return gmpsvm::engine_predict(*model->m, Xtest, m, out, nullptr, resolve(opt));
  });
}

int gmpsvm_train_csr(const int64_t* indptr, const int32_t* indices, const float* values, const int32_t* y, int64_t n,
                     int32_t d, int32_t k, double C, double gamma, double eps, const gmpsvm_options* opt,
                     gmpsvm_model** out) {
  return guarded([&]() {
    if (!out) throw Error(GMPSVM_EINVAL, "out is NULL");
    *out = nullptr;
    Model* m = nullptr;
    const int rc = gmpsvm::engine_train_csr(indptr, indices, values, y, n, d, k, C, gamma, eps, resolve(opt), &m);
    auto* h = new gmpsvm_model();
    h->m.reset(m);
    *out = h;
    return rc;
  });
}

int gmpsvm_predict_proba_csr(const gmpsvm_model* model, const int64_t* indptr, const int32_t* indices,
                             const float* values, int64_t m, double* out, const gmpsvm_options* opt) {
  return guarded([&]() {
    if (!model) throw Error(GMPSVM_EINVAL, "model is NULL");
    return gmpsvm::engine_predict_csr(*model->m, indptr, indices, values, m, out, resolve(opt));
  });
}

int gmpsvm_predict_proba(const gmpsvm_model* model, const float* Xtest, int64_t m, double* out) {
  return gmpsvm_predict_proba_ex(model, Xtest, m, out, nullptr);
}

int gmpsvm_predict_decision(const gmpsvm_model* model, const float* Xtest, int64_t m, double* dec_out,
                            const gmpsvm_options* opt) {
  return guarded([&]() {
    if (!model) throw Error(GMPSVM_EINVAL, "model is NULL");
    return gmpsvm::engine_predict(*model->m, Xtest, m, nullptr, dec_out, resolve(opt));
  });
}

void gmpsvm_model_free(gmpsvm_model* model) {
  try {
    delete model;
  } catch (...) {
  }
}

const char* gmpsvm_last_error(void) { return g_err.c_str(); }

int gmpsvm_model_dims(const gmpsvm_model* model, int32_t* k, int32_t* d, int64_t* n_sv, int32_t* n_pairs_trained) {
  return guarded([&]() {
    if (!model) throw Error(GMPSVM_EINVAL, "model is NULL");
    if (k) *k = model->m->k;
    if (d) *d = model->m->d;
    if (n_sv) *n_sv = (int64_t)model->m->sv_pos.size();
    if (n_pairs_trained) *n_pairs_trained = model->m->n_trained();
    return GMPSVM_OK;
  });
}

int gmpsvm_model_pair_iters(const gmpsvm_model* model, int32_t s, int32_t t, int64_t* outer, int64_t* inner,
                            int64_t* rows) {
  return guarded([&]() {
    if (!model) throw Error(GMPSVM_EINVAL, "model is NULL");
    const Model& m = *model->m;
    if (s < 0 || t <= s || t >= m.k) throw Error(GMPSVM_EINVAL, "need 0 <= s < t < k");
    const int p = gmpsvm::pair_index(s, t, m.k);
    auto at = [&](const std::vector<int64_t>& v) { return p < (int)v.size() ? v[p] : (int64_t)0; };
    if (outer) *outer = at(m.pair_outer);
    if (inner) *inner = at(m.pair_inner);
    if (rows) *rows = at(m.pair_rows);
    return GMPSVM_OK;
  });
}

int gmpsvm_model_pair(const gmpsvm_model* model, int32_t s, int32_t t, double* b, double* A, double* B,
                      double* alpha_out) {
  return guarded([&]() {
    if (!model) throw Error(GMPSVM_EINVAL, "model is NULL");
    const Model& m = *model->m;
    if (s < 0 || t <= s || t >= m.k) throw Error(GMPSVM_EINVAL, "need 0 <= s < t < k");
    const int p = gmpsvm::pair_index(s, t, m.k);
    if (!m.trained[p]) throw Error(GMPSVM_EINVAL, "pair not trained by this model");
    if (b) *b = m.b[p];
    if (A) *A = m.A[p];
    if (B) *B = m.B[p];
    if (alpha_out) {
      {
        std::lock_guard<std::mutex> lk(m.mu);
        gmpsvm::ensure_host_alpha(m);
      }
      const auto po = m.pair_offsets();
      std::copy(m.alpha.begin() + po[p], m.alpha.begin() + po[p + 1], alpha_out);
    }
    return m.status[p] & 0xff ? GMPSVM_WARN_MAXITER : GMPSVM_OK;
  });
}

int gmpsvm_model_sv_index(const gmpsvm_model* model, int64_t* idx_out) {
  return guarded([&]() {
    if (!model || !idx_out) throw Error(GMPSVM_EINVAL, "null argument");
    for (size_t i = 0; i < model->m->sv_pos.size(); ++i) idx_out[i] = model->m->perm[model->m->sv_pos[i]];
    return GMPSVM_OK;
  });
}

int gmpsvm_model_train_stats(const gmpsvm_model* model, gmpsvm_train_stats* stats) {
  return guarded([&]() {
    if (!model || !stats) throw Error(GMPSVM_EINVAL, "null argument");
    *stats = model->m->stats;
    return GMPSVM_OK;
  });
}

void gmpsvm_last_predict_stats(gmpsvm_predict_stats* stats) {
  if (stats) *stats = gmpsvm::tls_predict_stats();
}

int gmpsvm_model_serialize(const gmpsvm_model* model, void* buf, size_t* len) {
  return guarded([&]() {
    if (!model || !len) throw Error(GMPSVM_EINVAL, "null argument");
    const std::vector<uint8_t> blob = serialize(*model->m);
    const size_t cap = *len;
    *len = blob.size();
    if (!buf) return GMPSVM_OK;
    if (cap < blob.size()) throw Error(GMPSVM_EINVAL, "buffer too small");
    std::memcpy(buf, blob.data(), blob.size());
    return GMPSVM_OK;
  });
}

int gmpsvm_model_deserialize(const void* buf, size_t len, gmpsvm_model** out) {
  return guarded([&]() {
    if (!out) throw Error(GMPSVM_EINVAL, "out is NULL");
    *out = nullptr;
    auto* h = new gmpsvm_model();
    h->m.reset(deserialize(buf, len));
    *out = h;
    return GMPSVM_OK;
  });
}

int gmpsvm_model_merge(const gmpsvm_model* const* parts, int32_t n_parts, gmpsvm_model** out) {
  return guarded([&]() {
    if (!parts || !out || n_parts < 1) throw Error(GMPSVM_EINVAL, "bad merge arguments");
    *out = nullptr;
    std::vector<const Model*> ms(n_parts);
    for (int i = 0; i < n_parts; ++i) {
      if (!parts[i]) throw Error(GMPSVM_EINVAL, "null part");
      ms[i] = parts[i]->m.get();
    }
    std::unique_ptr<Model> m(merge(ms.data(), n_parts));
    auto* h = new gmpsvm_model();
    h->m = std::move(m);
    *out = h;
    return GMPSVM_OK;
  });
}

int gmpsvm_model_from_alpha(const float* X, const int32_t* y, int64_t n, int32_t d, int32_t k, double C, double gamma,
                            const double* alpha, const double* b, const double* A, const double* B,
                            const int32_t* status, const gmpsvm_options* opt, gmpsvm_model** out) {
  return guarded([&]() {
    if (!out) throw Error(GMPSVM_EINVAL, "out is NULL");
    *out = nullptr;
    Model* m = nullptr;
    const int rc = gmpsvm::engine_model_from_alpha(X, y, n, d, k, C, gamma, alpha, b, A, B, status, resolve(opt), &m);
    auto* h = new gmpsvm_model();
    h->m.reset(m);
    *out = h;
    return rc;
  });
}

int gmpsvm_rbf_kernel(const float* X, int64_t n, const float* Y, int64_t m, int32_t d, double gamma, float* K_out,
                      const gmpsvm_options* opt) {
  return guarded([&]() { return gmpsvm::engine_rbf_kernel(X, n, Y, m, d, gamma, K_out, resolve(opt)); });
}

int gmpsvm_couple(const double* dec, int64_t m, int32_t k, const double* A, const double* B, double* prob_out,
                  const gmpsvm_options* opt) {
  return guarded([&]() { return gmpsvm::engine_couple(dec, m, k, A, B, prob_out, resolve(opt)); });
}

struct gmpsvm_shard {
  gmpsvm::Shard* s = nullptr;
};

int gmpsvm_shard_create(const float* X, const int32_t* y, int64_t n, int32_t d, int32_t k, int32_t s, int32_t t,
                        double C, double gamma, double eps, int32_t rank, int32_t world, const gmpsvm_options* opt,
                        gmpsvm_shard** out) {
  return guarded([&]() {
    if (!out) throw Error(GMPSVM_EINVAL, "out is NULL");
    *out = nullptr;
    gmpsvm::Shard* sh = gmpsvm::shard_create(X, y, n, d, k, s, t, C, gamma, eps, rank, world, resolve(opt));
    *out = new gmpsvm_shard{sh};
    return GMPSVM_OK;
  });
}
int32_t gmpsvm_shard_cand_doubles(const gmpsvm_shard* sh) { return sh ? gmpsvm::shard_cand_doubles(sh->s) : 0; }
int gmpsvm_shard_slice(const gmpsvm_shard* sh, int64_t* lo, int64_t* hi, int64_t* n_p, int32_t* ws_size) {
  return guarded([&]() {
    if (!sh) throw Error(GMPSVM_EINVAL, "shard is NULL");
    gmpsvm::shard_slice(sh->s, lo, hi, n_p, ws_size);
    return GMPSVM_OK;
  });
}
int gmpsvm_shard_candidates(gmpsvm_shard* sh, double* out) {
  return guarded([&]() {
    if (!sh || !out) throw Error(GMPSVM_EINVAL, "null argument");
    gmpsvm::shard_candidates(sh->s, out);
    return GMPSVM_OK;
  });
}
int gmpsvm_shard_select(gmpsvm_shard* sh, const double* all, int32_t* stop, double* fws_out) {
  return guarded([&]() {
    if (!sh || !all || !stop) throw Error(GMPSVM_EINVAL, "null argument");
    return gmpsvm::shard_select(sh->s, all, stop, fws_out);
  });
}
int gmpsvm_shard_fws(gmpsvm_shard* sh, double* fws) {
  return guarded([&]() {
    if (!sh || !fws) throw Error(GMPSVM_EINVAL, "null argument");
    gmpsvm::shard_fws(sh->s, fws);
    return GMPSVM_OK;
  });
}
int gmpsvm_shard_step(gmpsvm_shard* sh, const double* fws_sum, double* cand_out) {
  return guarded([&]() {
    if (!sh || !fws_sum) throw Error(GMPSVM_EINVAL, "null argument");
    gmpsvm::shard_step(sh->s, fws_sum, cand_out);
    return GMPSVM_OK;
  });
}
int gmpsvm_shard_f(gmpsvm_shard* sh, double* f_slice) {
  return guarded([&]() {
    if (!sh || !f_slice) throw Error(GMPSVM_EINVAL, "null argument");
    gmpsvm::shard_f(sh->s, f_slice);
    return GMPSVM_OK;
  });
}
int gmpsvm_shard_finish(gmpsvm_shard* sh, const double* f_full, double* alpha, double* b, double* A, double* B,
                        int32_t* status, int64_t* outer_iters, int64_t* inner_iters) {
  return guarded([&]() {
    if (!sh || !f_full || !alpha || !b || !A || !B) throw Error(GMPSVM_EINVAL, "null argument");
    return gmpsvm::shard_finish(sh->s, f_full, alpha, b, A, B, status, outer_iters, inner_iters);
  });
}
void gmpsvm_shard_free(gmpsvm_shard* sh) {
  if (!sh) return;
  gmpsvm::shard_free(sh->s);
  delete sh;
}
int gmpsvm_shard_merge(const double* all, int32_t world, int32_t cand_doubles, int32_t need, int32_t need_u,
                       int32_t* picks_out, int32_t* n_picks, double* gap) {
  return guarded([&]() {
    if (!all || world < 1 || cand_doubles < 4 || need < 0 || need_u < 0 || need_u > need || !n_picks || !gap ||
        (need > 0 && !picks_out))
      throw Error(GMPSVM_EINVAL, "bad merge arguments");
    std::vector<int32_t> picks;
    *gap = gmpsvm::shard_merge(all, world, cand_doubles, need, need_u, picks);
    *n_picks = (int32_t)picks.size();
    for (size_t i = 0; i < picks.size(); ++i) picks_out[i] = picks[i];
    return GMPSVM_OK;
  });
}

uint64_t gmpsvm_launch_count(void) { return gmpsvm::g_launches.load(); }

int32_t gmpsvm_abi_version(void) { return GMPSVM_ABI_VERSION; }

}  // extern "C"
