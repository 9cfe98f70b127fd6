// stubs.cu -- placeholder TU (all four workloads are built).
