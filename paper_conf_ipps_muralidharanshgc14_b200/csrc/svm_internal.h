// svm_internal.h — host SVM model shared by svm.cpp and cv.cpp.
#pragma once
#include <stdint.h>

#include <vector>

namespace nitro {

struct SvmPair {
  int ca = 0, cb = 0;          // class indices (ca < cb); dec > 0 votes ca
  double rho = 0.0;
  std::vector<int> sv;         // training-sample ids
  std::vector<double> coef;    // y_i * alpha_i
};

struct SvmModel {
  int d = 0, n_train = 0;
  double gamma = 1.0;
  int const_label = -1;        // >= 0: single-class model
  std::vector<int> classes;    // ascending labels
  std::vector<double> X;       // training points [n_train * d] (SVs index into it)
  std::vector<SvmPair> pairs;
};

double rbf(const double *a, const double *b, int d, double gamma);
void svm_fit_impl(int n, int d, const double *X, const int *y, double C, double gamma, double tol, SvmModel &m);
void svm_decision_impl(const SvmModel &m, const double *x, std::vector<double> &dec);
int svm_predict_one(const SvmModel &m, const double *x);
void fold_assign_impl(int n, const int *y, int k, uint64_t seed, int *fold);
double cv_accuracy_impl(int n, int d, const double *X, const int *y, double C, double gamma, double tol, int folds,
                        uint64_t seed);

}  // namespace nitro
