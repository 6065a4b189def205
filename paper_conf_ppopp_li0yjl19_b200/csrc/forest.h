// Online batching-policy selector (§5, P272-274): a random forest over the features
// (mean M, mean N, mean K, batch size B) whose summed leaf vectors pick threshold or binary
// batching.  The trees are platform constants trained offline on B200 by
// scripts/train_forest.py from measured labels and emitted as forest_b200.h.
#pragma once
#include <stdint.h>

namespace vb {

struct ForestDef {
  int n_trees;
  const int32_t *root;        // [n_trees] node index of each tree's root
  const int8_t *feature;      // per node: 0 mean M, 1 mean N, 2 mean K, 3 B; -1 = leaf
  const double *threshold;    // per node: go left iff (double)(float)x[feature] <= threshold
  const int32_t *left, *right;
  const double *p_binary;     // per leaf: fraction of training samples labelled "binary"
};

// Features as the trees were trained on them: means over the batch in double, then float
// (sklearn evaluates trees on float32 inputs).
void forest_features(const int32_t *M, const int32_t *N, const int32_t *K, int batch, float x[4]);

// Sum the leaf vectors of all trees (P274) and return 1 (binary) if binary has the larger
// total, else 0 (threshold; ties go to threshold, the TLP-first heuristic).
int forest_select(const ForestDef &f, const float x[4]);

}  // namespace vb
