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
  double probA = 0.0, probB = 0.0;  // Platt sigmoid P(ca | f) = 1 / (1 + exp(A f + B))
};

struct SvmModel {
  int d = 0, n_train = 0;
  double gamma = 1.0;
  int const_label = -1;        // >= 0: single-class model
  std::vector<int> classes;    // ascending labels
  std::vector<double> X;       // training points [n_train * d] (SVs index into it)
  std::vector<SvmPair> pairs;
  bool prob = false;           // pairs carry Platt sigmoids
};

// Probability outputs (for BvSB active learning, P:L188 [20]): libSVM's method —
// per pair a Platt sigmoid fitted (Lin, Lin & Weng 2007 Newton) on decision
// values from an internal k-fold CV, then pairwise coupling (Wu, Lin & Weng
// 2004, method 2), solved exactly.
double sigmoid_predict(double f, double A, double B);
void sigmoid_train(int l, const double *dec, const int8_t *y, double &A, double &B);
void svm_fit_prob_impl(int n, int d, const double *X, const int *y, double C, double gamma, double tol, int folds,
                       uint64_t seed, SvmModel &m);
void svm_probability_impl(const SvmModel &m, const double *x, double *p /* [classes] */);

double rbf(const double *a, const double *b, int d, double gamma);
void svm_fit_impl(int n, int d, const double *X, const int *y, double C, double gamma, double tol, SvmModel &m);
void svm_decision_impl(const SvmModel &m, const double *x, std::vector<double> &dec);
int svm_predict_one(const SvmModel &m, const double *x);
void fold_assign_impl(int n, const int *y, int k, uint64_t seed, int *fold);
double cv_accuracy_impl(int n, int d, const double *X, const int *y, double C, double gamma, double tol, int folds,
                        uint64_t seed);

}  // namespace nitro
