// Pilot training on the GPU (§IV-D, §V: LeakyReLU, SGD, learning rate 0.01;
// DESIGN.md reading R19): minibatch SGD on the mean squared error over the feature
// layers, the MLP selected by the NN type and the output layer, in fp64 (the pilot's fp32
// weights widen exactly; export rounds back to fp32 for dyo_load_pilot).
//
// One step = forward (layer by layer, post-activations kept), the loss and dL/dy, then per layer
// from the output back: the LeakyReLU derivative, dW / db and the gradient of the layer's input,
// and finally every update (gradients are taken at the step's starting weights). Every sum runs
// in a fixed order, one output element per thread, so a step is deterministic; the layers are a
// few hundred thousand MACs, so these are plain fp64 CUDA-core loops (latency-bound, like K1).
#include <cuda_runtime.h>

#include <cstdint>
#include <cstring>
#include <vector>

#include "dyo_internal.h"

namespace {

constexpr double kSlope = 0.01;

struct TLayer {
  int in_len, out_len;
  int in_buf, in_off;              // input: buffer id (0 = X, 1 = feature concat, 2.. = layer outputs)
  int out_buf, out_off;            // output buffer id and column offset
  int act;
  double* W;                       // device out x in
  double* b;
  double* dW;
  double* db;
  size_t host_W, host_b;           // index into the host weight list (for export)
};

}  // namespace

struct dyo_trainer {
  int device = 0;
  int F = 0, O = 0, max_batch = 0, nn_type = 0;
  std::vector<TLayer> L;
  std::vector<std::vector<double>> host_w;     // every weight array of the desc, desc order
  std::vector<int> widths;                     // per buffer: row stride
  std::vector<double*> buf;                    // B x width activations per buffer
  std::vector<double*> dbuf;                   // B x width gradients per buffer
  double* T = nullptr;                         // B x O targets
  double* loss = nullptr;                      // 1
  std::vector<void*> owned;
};

namespace dyo {

__global__ void cvt_kernel(const float* __restrict__ a, double* __restrict__ b, int64_t n) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    b[i] = (double)a[i];
}

__global__ void fwd_kernel(const double* __restrict__ W, const double* __restrict__ bias, const double* __restrict__ in,
                           int in_w, int in_off, int in_len, double* __restrict__ out, int out_w, int out_off,
                           int out_len, int B, int act) {
  const int64_t n = (int64_t)B * out_len;
  for (int64_t idx = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; idx < n; idx += (int64_t)gridDim.x * blockDim.x) {
    const int bb = (int)(idx / out_len), o = (int)(idx % out_len);
    double v = bias[o];
    const double* w = W + (int64_t)o * in_len;
    const double* x = in + (int64_t)bb * in_w + in_off;
    for (int i = 0; i < in_len; ++i) v = fma(w[i], x[i], v);
    out[(int64_t)bb * out_w + out_off + o] = act ? (v > 0.0 ? v : kSlope * v) : v;
  }
}

// L = (1 / (B O)) sum (y - t)^2 (MSELoss, mean), dL/dy = 2 (y - t) / (B O) (one block,
// fixed-order reduction)
__global__ void loss_kernel(const double* __restrict__ y, const double* __restrict__ t, double* __restrict__ dy, int B,
                            int O, double* __restrict__ loss) {
  __shared__ double part[1024];
  double s = 0.0;
  const int64_t n = (int64_t)B * O;
  for (int64_t i = threadIdx.x; i < n; i += blockDim.x) {
    const double d = y[i] - t[i];
    dy[i] = 2.0 * d / (double)n;
    s = fma(d, d, s);
  }
  part[threadIdx.x] = s;
  __syncthreads();
  for (int w = blockDim.x / 2; w > 0; w >>= 1) {
    if ((int)threadIdx.x < w) part[threadIdx.x] += part[threadIdx.x + w];
    __syncthreads();
  }
  if (threadIdx.x == 0) *loss = part[0] / (double)n;
}

// gradient w.r.t. the pre-activation: times LeakyReLU'(v) (sign of the post-activation)
__global__ void act_bwd_kernel(double* __restrict__ d, const double* __restrict__ a, int w, int off, int len, int B) {
  const int64_t n = (int64_t)B * len;
  for (int64_t idx = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; idx < n; idx += (int64_t)gridDim.x * blockDim.x) {
    const int bb = (int)(idx / len), o = (int)(idx % len);
    const int64_t k = (int64_t)bb * w + off + o;
    if (!(a[k] > 0.0)) d[k] *= kSlope;
  }
}

// dW[o][i] = sum_b dV[b][o] x[b][i]; db[o] = sum_b dV[b][o]
__global__ void grad_w_kernel(const double* __restrict__ dv, int dv_w, int dv_off, int out_len,
                              const double* __restrict__ in, int in_w, int in_off, int in_len, int B,
                              double* __restrict__ dW, double* __restrict__ db) {
  const int64_t n = (int64_t)out_len * (in_len + 1);
  for (int64_t idx = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; idx < n; idx += (int64_t)gridDim.x * blockDim.x) {
    const int o = (int)(idx / (in_len + 1)), i = (int)(idx % (in_len + 1));
    double s = 0.0;
    if (i < in_len) {
      for (int bb = 0; bb < B; ++bb) s = fma(dv[(int64_t)bb * dv_w + dv_off + o], in[(int64_t)bb * in_w + in_off + i], s);
      dW[(int64_t)o * in_len + i] = s;
    } else {
      for (int bb = 0; bb < B; ++bb) s += dv[(int64_t)bb * dv_w + dv_off + o];
      db[o] = s;
    }
  }
}

// dIn[b][i] = sum_o W[o][i] dV[b][o]
__global__ void grad_in_kernel(const double* __restrict__ W, const double* __restrict__ dv, int dv_w, int dv_off,
                               int out_len, double* __restrict__ din, int din_w, int din_off, int in_len, int B) {
  const int64_t n = (int64_t)B * in_len;
  for (int64_t idx = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; idx < n; idx += (int64_t)gridDim.x * blockDim.x) {
    const int bb = (int)(idx / in_len), i = (int)(idx % in_len);
    double s = 0.0;
    for (int o = 0; o < out_len; ++o) s = fma(W[(int64_t)o * in_len + i], dv[(int64_t)bb * dv_w + dv_off + o], s);
    din[(int64_t)bb * din_w + din_off + i] = s;
  }
}

__global__ void sgd_kernel(double* __restrict__ p, const double* __restrict__ g, int64_t n, double lr) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    p[i] -= lr * g[i];
}

static int grid_for(int64_t n) {
  const int64_t g = (n + 255) / 256;
  return (int)(g < 1184 ? (g < 1 ? 1 : g) : 1184);
}

}  // namespace dyo

using namespace dyo;

extern "C" {

dyo_status dyo_trainer_create(const dyo_pilot_desc* w, int32_t nn_type, int32_t max_batch, int32_t device,
                              dyo_trainer** out) {
  if (!w || !out || nn_type < 0 || nn_type > 2 || max_batch < 1 || w->n_mlp < 1 || w->F < 1 || w->O < 1)
    return DYO_E_INVAL;
  if (cudaSetDevice(device) != cudaSuccess) return DYO_E_CUDA;
  dyo_trainer* tr = new dyo_trainer();
  tr->device = device;
  tr->F = w->F;
  tr->O = w->O;
  tr->max_batch = max_batch;
  tr->nn_type = nn_type;
  auto keep = [&](const float* p, size_t n) {
    tr->host_w.emplace_back(p, p + n);
    return tr->host_w.size() - 1;
  };
  // buffers: 0 = X (F wide), 1 = feature concat, 2 + l = output of MLP layer l, last = logits
  int concat = 0;
  for (int i = 0; i < w->n_feature; ++i) concat += w->feat_out[i];
  tr->widths = {w->F, std::max(concat, 1)};
  for (int l = 0; l < w->n_mlp; ++l) tr->widths.push_back(w->mlp_out[l]);
  tr->widths.push_back(w->O);
  const int out_buf = (int)tr->widths.size() - 1;
  size_t idx_feat = 0;
  int off = 0;
  for (int i = 0; i < w->n_feature; ++i) {
    TLayer L{};
    L.in_len = w->feat_len[i]; L.out_len = w->feat_out[i];
    L.in_buf = 0; L.in_off = w->feat_off[i]; L.out_buf = 1; L.out_off = off; L.act = 1;
    L.host_W = keep(w->feat_W[i], (size_t)L.out_len * L.in_len);
    L.host_b = keep(w->feat_b[i], (size_t)L.out_len);
    off += L.out_len;
    tr->L.push_back(L);
    ++idx_feat;
  }
  std::vector<size_t> mlp_hw, mlp_hb;
  for (int k = 0; k < 3; ++k)
    for (int l = 0; l < w->n_mlp; ++l) {
      mlp_hw.push_back(keep(w->mlp_W[k * w->n_mlp + l], (size_t)w->mlp_out[l] * w->mlp_in[l]));
      mlp_hb.push_back(keep(w->mlp_b[k * w->n_mlp + l], (size_t)w->mlp_out[l]));
    }
  for (int l = 0; l < w->n_mlp; ++l) {
    TLayer L{};
    L.in_len = w->mlp_in[l]; L.out_len = w->mlp_out[l];
    L.in_buf = l == 0 ? (w->n_feature ? 1 : 0) : 2 + (l - 1); L.in_off = 0;
    L.out_buf = 2 + l; L.out_off = 0; L.act = 1;
    L.host_W = mlp_hw[(size_t)nn_type * w->n_mlp + l];
    L.host_b = mlp_hb[(size_t)nn_type * w->n_mlp + l];
    tr->L.push_back(L);
  }
  {
    TLayer L{};
    L.in_len = w->out_in; L.out_len = w->O;
    L.in_buf = 2 + w->n_mlp - 1; L.in_off = 0; L.out_buf = out_buf; L.out_off = 0; L.act = 0;
    L.host_W = keep(w->out_W, (size_t)w->O * w->out_in);
    L.host_b = keep(w->out_b, (size_t)w->O);
    tr->L.push_back(L);
  }
  auto dal = [&](double** p, size_t n) {
    if (cudaMalloc(p, std::max<size_t>(n, 1) * sizeof(double)) != cudaSuccess) return false;
    tr->owned.push_back(*p);
    return true;
  };
  bool ok = true;
  for (auto& L : tr->L) {
    const size_t nw = (size_t)L.out_len * L.in_len;
    ok = ok && dal(&L.W, nw) && dal(&L.b, L.out_len) && dal(&L.dW, nw) && dal(&L.db, L.out_len);
    if (ok) {
      ok = cudaMemcpy(L.W, tr->host_w[L.host_W].data(), nw * 8, cudaMemcpyHostToDevice) == cudaSuccess &&
           cudaMemcpy(L.b, tr->host_w[L.host_b].data(), (size_t)L.out_len * 8, cudaMemcpyHostToDevice) == cudaSuccess;
    }
  }
  for (int wd : tr->widths) {
    double *a = nullptr, *d = nullptr;
    ok = ok && dal(&a, (size_t)max_batch * wd) && dal(&d, (size_t)max_batch * wd);
    tr->buf.push_back(a);
    tr->dbuf.push_back(d);
  }
  ok = ok && dal(&tr->T, (size_t)max_batch * w->O) && dal(&tr->loss, 1);
  if (!ok) {
    dyo_trainer_destroy(tr);
    return DYO_E_NOMEM;
  }
  *out = tr;
  return DYO_OK;
}

dyo_status dyo_trainer_destroy(dyo_trainer* tr) {
  if (!tr) return DYO_E_INVAL;
  cudaSetDevice(tr->device);
  cudaDeviceSynchronize();
  for (void* p : tr->owned) cudaFree(p);
  delete tr;
  return DYO_OK;
}

dyo_status dyo_trainer_step(dyo_trainer* tr, const float* feat, const float* target, int32_t B, double lr,
                            double* loss, void* stream) {
  if (!tr || !feat || !target || B < 1 || B > tr->max_batch) return DYO_E_INVAL;
  if (cudaSetDevice(tr->device) != cudaSuccess) return DYO_E_CUDA;
  cudaStream_t s = (cudaStream_t)stream;
  const int64_t nx = (int64_t)B * tr->F, nt = (int64_t)B * tr->O;
  cvt_kernel<<<grid_for(nx), 256, 0, s>>>(feat, tr->buf[0], nx);
  cvt_kernel<<<grid_for(nt), 256, 0, s>>>(target, tr->T, nt);
  const auto& Wd = tr->widths;
  for (const auto& L : tr->L)
    fwd_kernel<<<grid_for((int64_t)B * L.out_len), 256, 0, s>>>(L.W, L.b, tr->buf[L.in_buf], Wd[L.in_buf], L.in_off,
                                                                L.in_len, tr->buf[L.out_buf], Wd[L.out_buf], L.out_off,
                                                                L.out_len, B, L.act);
  const int ob = (int)Wd.size() - 1;
  loss_kernel<<<1, 1024, 0, s>>>(tr->buf[ob], tr->T, tr->dbuf[ob], B, tr->O, tr->loss);
  // backward: output layer first; a layer's input gradient goes to its input buffer's gradient
  // (feature layers share the concat buffer at their column offsets; X needs none)
  for (int li = (int)tr->L.size() - 1; li >= 0; --li) {
    const TLayer& L = tr->L[li];
    double* dv = tr->dbuf[L.out_buf];
    if (L.act)
      act_bwd_kernel<<<grid_for((int64_t)B * L.out_len), 256, 0, s>>>(dv, tr->buf[L.out_buf], Wd[L.out_buf], L.out_off,
                                                                       L.out_len, B);
    grad_w_kernel<<<grid_for((int64_t)L.out_len * (L.in_len + 1)), 256, 0, s>>>(
        dv, Wd[L.out_buf], L.out_off, L.out_len, tr->buf[L.in_buf], Wd[L.in_buf], L.in_off, L.in_len, B, L.dW, L.db);
    if (L.in_buf != 0)
      grad_in_kernel<<<grid_for((int64_t)B * L.in_len), 256, 0, s>>>(L.W, dv, Wd[L.out_buf], L.out_off, L.out_len,
                                                                     tr->dbuf[L.in_buf], Wd[L.in_buf], L.in_off, L.in_len, B);
  }
  for (const auto& L : tr->L) {
    const int64_t nw = (int64_t)L.out_len * L.in_len;
    sgd_kernel<<<grid_for(nw), 256, 0, s>>>(L.W, L.dW, nw, lr);
    sgd_kernel<<<grid_for(L.out_len), 256, 0, s>>>(L.b, L.db, L.out_len, lr);
  }
  if (cudaGetLastError() != cudaSuccess) return DYO_E_CUDA;
  if (loss) {
    if (cudaMemcpyAsync(loss, tr->loss, 8, cudaMemcpyDeviceToHost, s) != cudaSuccess) return DYO_E_CUDA;
    if (cudaStreamSynchronize(s) != cudaSuccess) return DYO_E_CUDA;
  }
  return DYO_OK;
}

dyo_status dyo_trainer_export(dyo_trainer* tr, double* blob, int64_t cap, int64_t* n) {
  if (!tr || !n) return DYO_E_INVAL;
  if (cudaSetDevice(tr->device) != cudaSuccess || cudaDeviceSynchronize() != cudaSuccess) return DYO_E_CUDA;
  for (const auto& L : tr->L) {
    if (cudaMemcpy(tr->host_w[L.host_W].data(), L.W, (size_t)L.out_len * L.in_len * 8, cudaMemcpyDeviceToHost) != cudaSuccess ||
        cudaMemcpy(tr->host_w[L.host_b].data(), L.b, (size_t)L.out_len * 8, cudaMemcpyDeviceToHost) != cudaSuccess)
      return DYO_E_CUDA;
  }
  int64_t tot = 0;
  for (const auto& v : tr->host_w) tot += (int64_t)v.size();
  *n = tot;
  if (!blob) return DYO_OK;
  if (cap < tot) return DYO_E_CAPACITY;
  int64_t o = 0;
  for (const auto& v : tr->host_w) {
    std::memcpy(blob + o, v.data(), v.size() * 8);
    o += (int64_t)v.size();
  }
  return DYO_OK;
}

}  // extern "C"
