// Random-forest policy selector (PAPER.md P272-274); see forest.h.
#include "forest.h"

namespace vb {

void forest_features(const int32_t *M, const int32_t *N, const int32_t *K, int batch, float x[4]) {
  double sm = 0, sn = 0, sk = 0;
  for (int i = 0; i < batch; ++i) {
    sm += M[i];
    sn += N[i];
    sk += K[i];
  }
  const double b = batch > 0 ? (double)batch : 1.0;
  x[0] = (float)(sm / b);
  x[1] = (float)(sn / b);
  x[2] = (float)(sk / b);
  x[3] = (float)batch;
}

int forest_select(const ForestDef &f, const float x[4]) {
  double p_bin = 0, p_thr = 0;
  for (int t = 0; t < f.n_trees; ++t) {
    int n = f.root[t];
    while (f.feature[n] >= 0) n = ((double)x[f.feature[n]] <= f.threshold[n]) ? f.left[n] : f.right[n];
    p_bin += f.p_binary[n];
    p_thr += 1.0 - f.p_binary[n];
  }
  return p_bin > p_thr ? 1 : 0;
}

}  // namespace vb
